"""GPU parity of the SURVEY §8(f) rows f1 and f2 on the device.

* f2: plans scheduled by the round-robin baseline (``sched=rr``)
  give different sub-pipelines, lane lists and orders than HPDS.  A wrong order could
  deadlock or race on the device, so they run here -- staged and direct transports,
  register and TMA paths -- against the oracle's replay of the oracle's own RR plan.
* f1: the paper's Fig. 16 program text (``tests/golden``) is loaded
  verbatim (only nNodes / nGpusperNode / nRanks / GPUPerNode instantiated for 8 ranks)
  through ``rescclLoadAlgorithm``: the C++ ResCCLang front end, planner and generated
  kernel run it, and the result must equal the oracle's replay of its own transcription
  of the listing (``oracle.ir.hm_allreduce``) byte for byte.
"""
import os

import numpy as np
import pytest

import resccl_inputs as inp
from gpu_helpers import run_virtual
from oracle import dag, definition, hpds, ir as oir, lower, replay

pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden")

RR_CASES = [
    ("dbt", "allreduce", 8, {}), ("hm", "allreduce", 8, {"g": 4}), ("hm", "allgather", 8, {"g": 4}),
    ("synth", "allgather", 8, {"seed": 0, "fanout": 2}), ("synth", "reducescatter", 8, {"seed": 1, "fanout": 3}),
    ("ring", "allreduce", 8, {}),
]


def _rr_expect(g, xs, dtype, count, cb, inst, K, direct):
    edges, _ = dag.build_dag(g)
    pl = lower.lower(g, "pair", Pr=hpds.round_robin(g, edges, "pair"), direct=direct)
    return replay.replay(pl, xs, dtype, count, chunk_bytes=cb, instances=inst, K=K)


def _check(outs, exp):
    for r in range(len(outs)):
        assert np.array_equal(outs[r].view(np.uint8), exp[r].view(np.uint8)), f"rank {r}"


@pytest.mark.timeout(300)
@pytest.mark.parametrize("name,coll,n,kw", RR_CASES)
@pytest.mark.parametrize("direct", [0, 1])
def test_round_robin_plans_bit_exact(name, coll, n, kw, direct):
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    g = oir.generate(name, coll, n, **kw)
    count = 3 * 4096 + 77
    for k, v in dict(sched="rr", chunkbytes=4096, instances=2, fifodepth=2, direct=direct).items():
        g.extra[k] = str(v)
    m = count * n if coll == "reducescatter" else count
    xs = inp.all_inputs("bfloat16", 21, n, m)
    outs, info, err = run_virtual(R, g.to_text(), coll, xs, "bfloat16", count)
    assert err == 0 and info["sched"] == "rr"
    _check(outs, _rr_expect(g, xs, "bfloat16", count, 4096, 2, 2, bool(direct)))


@pytest.mark.timeout(300)
@pytest.mark.parametrize("name,coll,kw", [("dbt", "allreduce", {}), ("hm", "allreduce", {"g": 4}),
                                          ("synth", "reducescatter", {"seed": 0, "fanout": 2})])
def test_round_robin_plans_tma_path(name, coll, kw):
    """Instance slices above tmamin: the TMA lane engine runs the RR lane lists."""
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    g = oir.generate(name, coll, n, **kw)
    count = (2 << 20) + 4099
    for k, v in dict(sched="rr", chunkbytes=1 << 20, instances=2, fifodepth=2, direct=1).items():
        g.extra[k] = str(v)
    m = count * n if coll == "reducescatter" else count
    xs = inp.all_inputs("float32", 22, n, m)
    outs, info, err = run_virtual(R, g.to_text(), coll, xs, "float32", count)
    assert err == 0
    _check(outs, _rr_expect(g, xs, "float32", count, 1 << 20, 2, 2, True))


def _fig16_text(n_nodes, gpn):
    src = open(os.path.join(GOLD, "fig16_hm_allreduce.py.txt")).read()
    src = src.replace("nRanks =32", f"nRanks ={n_nodes * gpn}").replace("GPUPerNode =8", f"GPUPerNode ={gpn}")
    src = src.replace("    nNodes = 4\n", f"    nNodes = {n_nodes}\n")
    return src.replace("    nGpusperNode = 8\n", f"    nGpusperNode = {gpn}\n")


@pytest.mark.timeout(300)
@pytest.mark.parametrize("dtype", ["bfloat16", "int32"])
def test_fig16_program_text_on_gpu(dtype):
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    text = _fig16_text(2, 4)
    assert text.lstrip("#").find("def ResCCLAlgo") >= 0
    n, count = 8, (3 << 20) + 1001
    xs = inp.all_inputs(dtype, 23, n, count)
    outs, info, err = run_virtual(R, text, "allreduce", xs, dtype, count)
    assert err == 0
    assert info["instances"] == 4 and info["nwarps"] == 16   # nChannels=4, nWarps=16 (Fig. 16 header)
    assert info["ctas"] == [4] * n                            # Table 3 Topo1: 8 lanes = 4 duplex CTAs
    g = oir.hm_allreduce(2, 4)
    exp = replay.replay(lower.lower(g), xs, dtype, count, chunk_bytes=1 << 20, instances=4, K=4)
    _check(outs, exp)
    if dtype == "int32":
        _check(outs, definition.allreduce(xs, "int32"))


@pytest.mark.timeout(300)
@pytest.mark.parametrize("name,coll,kw", [("ring", "allreduce", {}), ("hm", "allreduce", {"g": 4}),
                                          ("dbt", "allreduce", {})])
def test_tb_utilization_trace(name, coll, kw):
    """Table 3 instrumentation (trace=1): per-lane (the paper's TB)
    and per-CTA idle ratios are well-formed, one lane record per traced lane, and tracing
    leaves the result bit-exact."""
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    g = oir.generate(name, coll, n, **kw)
    count = (1 << 20) + 333
    for k, v in dict(chunkbytes=1 << 18, instances=2, fifodepth=2, direct=1, trace=1, nwarps=8).items():
        g.extra[k] = str(v)
    xs = inp.all_inputs("float32", 24, n, count)
    grp = R.VirtualGroup(n, 0)
    try:
        import torch
        from gpu_helpers import to_numpy, to_torch
        grp.load(g.to_text())
        info = grp.plan_info()
        s = [to_torch(x, "float32") for x in xs]
        r = [torch.empty_like(t) for t in s]
        grp.allreduce(s, r)
        torch.cuda.synchronize()
        assert grp.async_error() == 0
        u = R.rescclGetTbUtilization(grp.comms[0].algos[-1])
        outs = [to_numpy(t, "float32") for t in r]
    finally:
        grp.destroy()
    lanes = sum(len(a) > 0 for rk in info["plan"]["ranks"] for c in rk["ctas"] for a in (c["send"], c["recv"]))
    assert u["tbs"] == lanes * info["instances"]
    assert u["ctas"] == sum(info["blocks_per_rank"])
    for k in ("comm_time", "avg_idle", "max_idle", "cta_comm_time", "cta_avg_idle", "cta_max_idle"):
        assert 0.0 <= u[k] <= 1.0, (k, u[k])
    exp = replay.replay(lower.lower(g, direct=True), xs, "float32", count, chunk_bytes=1 << 18, instances=2, K=2)
    _check(outs, exp)


@pytest.mark.timeout(300)
def test_size_based_algorithm_selection():
    """minbytes / maxbytes (include/resccl.h): a full-mesh AllReduce (HM with one node of 8,
    Fig. 16 at nNodes = 1) serves small calls, the ring large ones; every call is bit-exact
    against the oracle's replay of the algorithm that served it (the two reduce in
    different association orders, so a wrong pick shows up as a byte difference)."""
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    from gpu_helpers import to_numpy, to_torch
    n = 8
    mesh = oir.generate("hm", "allreduce", n, g=8)
    ring = oir.generate("ring", "allreduce", n)
    mesh.extra.update(dict(instances="2", chunkbytes=str(1 << 20), direct="1", maxbytes=str(256 << 10)))
    ring.extra.update(dict(instances="4", chunkbytes=str(1 << 20), direct="1", minbytes=str((256 << 10) + 1)))
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(ring.to_text())
        grp.load(mesh.to_text())
        for count, g, inst in ((1000, mesh, 2), (64 << 10, mesh, 2), ((64 << 10) + 8, ring, 4), (1 << 20, ring, 4)):
            xs = inp.all_inputs("float32", 30, n, count)
            s = [to_torch(x, "float32") for x in xs]
            r = [torch.empty_like(t) for t in s]
            grp.allreduce(s, r)
            torch.cuda.synchronize()
            assert grp.async_error() == 0
            exp = replay.replay(lower.lower(g, direct=True), xs, "float32", count, chunk_bytes=1 << 20,
                                instances=inst, K=4)
            _check([to_numpy(t, "float32") for t in r], exp)
    finally:
        grp.destroy()


@pytest.mark.timeout(300)
@pytest.mark.parametrize("name,coll,kw", [("ring", "allreduce", {}), ("hm", "allreduce", {"g": 4}),
                                          ("dbt", "allreduce", {}), ("synth", "reducescatter", {"seed": 1, "fanout": 3}),
                                          ("ring", "allgather", {}), ("hm", "allreduce", {"g": 8})])
@pytest.mark.parametrize("count,cb", [(3 * 4096 + 77, 4096), ((2 << 20) + 4099, 1 << 20)])
def test_pushreduce_bit_exact(name, coll, kw, count, cb):
    """Push-reduce variant of the direct transport (R31): the sender pushes
    rrc operands into the receiver's FIFO slot (staged) while recv payloads are pushed
    straight into the receiver's location; register path and TMA engine."""
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    g = oir.generate(name, coll, n, **kw)
    for k, v in dict(chunkbytes=cb, instances=2, fifodepth=2, direct=1, pushreduce=1).items():
        g.extra[k] = str(v)
    m = count * n if coll == "reducescatter" else count
    xs = inp.all_inputs("float32", 25, n, m)
    outs, info, err = run_virtual(R, g.to_text(), coll, xs, "float32", count)
    assert err == 0 and info["pushreduce"] == 1
    exp = replay.replay(lower.lower(g, direct=True, pushreduce=True), xs, "float32", count, chunk_bytes=cb,
                        instances=2, K=2)
    _check(outs, exp)
