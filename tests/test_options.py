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
