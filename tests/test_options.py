"""Host-side option handling of the planner/codegen (no GPU): defaults and auto values
reported in the plan JSON, environment overrides, and NVRTC builds of every kernel
variant the options select (device epochs on/off, bulk reduction, cpoll)."""
import os

import pytest

import paper_conf_sigcomm_liuhlgcwz025_b200 as R


def test_defaults_and_auto_values():
    ar = R.rescclPlanIr(R.rescclGenerateIr("ring", "allreduce", 4))
    ag = R.rescclPlanIr(R.rescclGenerateIr("ring", "allgather", 4))
    assert ar["devepoch"] == 1 and ag["devepoch"] == 1
    assert ar["bulkred"] == 1 and ag["bulkred"] == 0  # auto: on for AllReduce only
    assert ar["tmatile"] == 24576 and ar["tmastages"] == 2
    assert R.rescclPlanIr(R.rescclGenerateIr("ring", "allreduce", 4), "bulkred=0 devepoch=0")["bulkred"] == 0


def test_environment_override(monkeypatch):
    monkeypatch.setenv("RESCCL_DEVEPOCH", "0")
    assert R.rescclPlanIr(R.rescclGenerateIr("ring", "allreduce", 4))["devepoch"] == 0


@pytest.mark.parametrize("opts", ["devepoch=0", "devepoch=1", "bulkred=1 direct=1", "bulkred=0", "cpoll=1",
                                  "tmamin=1073741824", "ring=1"])
def test_kernel_variants_build(opts):
    text = R.rescclGenerateIr("ring", "allreduce", 4)
    for dt in (R.rescclBfloat16, R.rescclFloat32):
        assert R.rescclCompileIr(text, opts + " instances=2", dt, R.rescclSum) > 0


def test_generated_source_uses_device_epochs():
    src = R.rescclCodegenIr(R.rescclGenerateIr("ring", "allreduce", 2), "instances=1")
    assert "epochs_begin" in src and "epochs_end" in src


@pytest.mark.parametrize("opts", ["splitfence=0", "splitfence=1", "postgroup=0", "postgroup=1 direct=1", "earlyexit=0"])
def test_fence_and_post_group_variants_build(opts):
    """both fence variants and both post forms compile for sm_100a."""
    text = R.rescclGenerateIr("hm", "allreduce", 8, "g=8")
    assert R.rescclCompileIr(text, opts + " linkmodel=port instances=1", R.rescclBfloat16, R.rescclSum) > 0


def _calls(src):
    import re
    single = [int(m) for m in re.findall(r"L\.pidx = (\d+);[^\n]*rdev::run<", src)]
    groups = [[int(x) for x in g.split(",")] for g in re.findall(r"static __constant__ int kPg\[\d+\] = \{([^}]*)\}", src)]
    return single, groups


def test_post_group_covers_every_primitive_once():
    """The full mesh's send lane starts with N-1 dependency-free pull-sends: with postgroup=1
    they become one grouped call, and every primitive of the plan is still called exactly
    once per lane (no primitive dropped or duplicated); postgroup=0 or the ring (one pull-send
    per lane) emit no group."""
    text = R.rescclGenerateIr("hm", "allreduce", 8, "g=8")
    opts = "linkmodel=port instances=1 direct=1"
    plan = R.rescclPlanIr(text, opts)["plan"]
    for pg in (1, 0):
        src = R.rescclCodegenIr(text, opts + f" postgroup={pg}")
        single, groups = _calls(src)
        if pg:
            assert len(groups) == 8 and all(len(g) == 7 for g in groups)
            for r, g in enumerate(groups):
                assert all(plan["ranks"][r]["prims"][k]["kind"] == "psend" for k in g)
        else:
            assert not groups
        total = len(single) + sum(len(g) for g in groups)
        assert total == sum(len(rp["prims"]) for rp in plan["ranks"])
    ring = R.rescclCodegenIr(R.rescclGenerateIr("ring", "allreduce", 8), "instances=1 direct=1")
    assert "run_post_group" not in ring


def test_split_fence_macro():
    text = R.rescclGenerateIr("ring", "allreduce", 4)
    assert "#define RESCCL_SPLIT_FENCE 1" in R.rescclCodegenIr(text, "")
    assert "#define RESCCL_SPLIT_FENCE 0" in R.rescclCodegenIr(text, "splitfence=0")


def test_one_warp_lanes_take_the_register_path():
    """nwarps=2 leaves no combine warp beside a lane's leader: the TMA engine is switched off
    (its 'combined' barriers would count zero arrivals and never complete)."""
    text = R.rescclGenerateIr("hm", "allreduce", 8, "g=8")
    assert R.rescclPlanIr(text, "nwarps=2 instances=1")["tma"] == 0
    assert R.rescclPlanIr(text, "nwarps=4 instances=1")["tma"] == 1
