"""Host-side product path (C++ planner behind the C ABI) vs the independent oracle.

The C++ generators, DAG builder, HPDS scheduler, TB allocator and fusion pass must
produce exactly what the oracle (written separately from the same paper passages)
produces.  No GPU needed."""
import ctypes
import os
import re

import pytest

import paper_conf_sigcomm_liuhlgcwz025_b200 as R
from oracle import dag, hpds, ir as oir, lower, replay

CASES = [
    ("ring", "allreduce", 2, {}), ("ring", "allreduce", 3, {}), ("ring", "allreduce", 8, {}),
    ("ring", "allgather", 4, {}), ("ring", "allgather", 8, {}), ("ring", "reducescatter", 8, {}),
    ("ring", "allreduce", 16, {}),
    ("dbt", "allreduce", 4, {}), ("dbt", "allreduce", 8, {}), ("dbt", "allreduce", 6, {}),
    ("dbt", "allreduce", 7, {}), ("dbt", "allreduce", 16, {}),
    ("hm", "allreduce", 8, {"g": 4}), ("hm", "allreduce", 16, {"g": 8}), ("hm", "allreduce", 16, {"g": 4}),
    ("hm", "allgather", 8, {"g": 4}), ("hm", "allgather", 16, {"g": 8}),
    ("synth", "allgather", 8, {"seed": 0, "fanout": 2}), ("synth", "allgather", 8, {"seed": 5, "fanout": 3}),
    ("synth", "reducescatter", 8, {"seed": 1, "fanout": 2}),
    ("synth", "reducescatter", 8, {"seed": 7, "fanout": 3}),
]


def _oracle_ir(name, coll, n, kw):
    return oir.generate(name, coll, n, **kw)


def _cpp_ir(name, coll, n, kw):
    opts = " ".join(f"{k}={v}" for k, v in kw.items())
    return R.rescclGenerateIr(name, coll, n, opts)


@pytest.mark.parametrize("name,coll,n,kw", CASES)
def test_generators_match(name, coll, n, kw):
    a = _oracle_ir(name, coll, n, kw)
    b = oir.parse_text(_cpp_ir(name, coll, n, kw))
    assert (a.name, a.coll, a.nranks, a.nchunks) == (b.name, b.coll, b.nranks, b.nchunks)
    assert sorted(a.transfers) == sorted(b.transfers)
    assert a.extra == b.extra


def _norm_oracle(pl):
    tasks = pl.ir.transfers
    out = []
    for r in range(pl.ir.nranks):
        prims = pl.prims[r]

        def key(p):
            return (p.kind, p.chunk, p.pc,
                    tuple(tasks[p.recv_task]) if p.recv_task is not None else None,
                    tuple(tasks[p.send_task]) if p.send_task is not None else None,
                    p.src_buf or "none", p.dst_buf or "none", p.has_counter, p.rem_buf or "none")

        ctas = []
        for sl, rl in pl.lanes[r]:
            ctas.append(tuple(
                tuple((key(prims[i]), tuple(sorted(key(prims[d]) for d in prims[i].deps)),
                       tuple(sorted(key(prims[d]) for d in prims[i].ack_deps))) for i in lane)
                for lane in (sl, rl)))
        out.append(dict(
            ctas=ctas, n_conn=pl.n_connections[r], paper_tbs=pl.paper_tbs(r),
            send_groups=[[c[0] for c in g] for g in pl.send_groups[r]],
            recv_groups=[[c[0] for c in g] for g in pl.recv_groups[r]]))
    return out


def _norm_cpp(js):
    plan = js["plan"]
    tasks = [tuple(t) for t in plan["tasks"]]
    out = []
    for rp in plan["ranks"]:
        prims = rp["prims"]

        def key(p):
            return (p["kind"], p["chunk"], p["pc"],
                    tasks[p["recv_task"]] if p["recv_task"] >= 0 else None,
                    tasks[p["send_task"]] if p["send_task"] >= 0 else None,
                    p["src"], p["dst"], p["counter"], p["rem"])

        ctas = []
        for c in rp["ctas"]:
            ctas.append(tuple(
                tuple((key(prims[i]), tuple(sorted(key(prims[d]) for d in prims[i]["deps"])),
                       tuple(sorted(key(prims[d]) for d in prims[i]["ack_deps"]))) for i in lane)
                for lane in (c["send"], c["recv"])))
        out.append(dict(ctas=ctas, n_conn=rp["n_connections"], paper_tbs=rp["paper_tbs"],
                        send_groups=rp["send_groups"], recv_groups=rp["recv_groups"]))
    return out


@pytest.mark.parametrize("name,coll,n,kw", CASES)
@pytest.mark.parametrize("model", ["pair", "port"])
@pytest.mark.parametrize("fuse", [1, 0])
def test_plan_matches_oracle(name, coll, n, kw, model, fuse):
    g = _oracle_ir(name, coll, n, kw)
    text = g.to_text()
    js = R.rescclPlanIr(text, f"linkmodel={model} fuse={fuse}")
    pl = lower.lower(g, model, fuse=bool(fuse))
    # sub-pipelines: identical membership and insertion order
    tasks = [tuple(t) for t in js["plan"]["tasks"]]
    assert [[tasks[i] for i in pc] for pc in js["plan"]["Pr"]] == \
        [[tuple(g.transfers[i]) for i in pc] for pc in pl.Pr]
    assert js["plan"]["n_edges"] == len(pl.edges)
    assert js["plan"]["fused"] == pl.fused
    assert _norm_cpp(js) == _norm_oracle(pl)


def test_round_robin_not_exposed_but_hpds_table3():
    """C++ planner reproduces Table 3's expert #TB too."""
    for (nn, g, want) in ((2, 4, 8), (2, 8, 16), (4, 4, 8), (4, 8, 16)):
        for coll in ("allreduce", "allgather"):
            text = R.rescclGenerateIr("hm", coll, nn * g, f"g={g}")
            js = R.rescclPlanIr(text, "fuse=0")
            assert all(rp["paper_tbs"] == want for rp in js["plan"]["ranks"])


@pytest.mark.parametrize("name,coll,n,kw", CASES[:14])
def test_cpp_deadlock_check_agrees_with_oracle(name, coll, n, kw):
    g = _oracle_ir(name, coll, n, kw)
    text = g.to_text()
    for fuse in (0, 1):
        pl = lower.lower(g, "pair", fuse=bool(fuse))
        for K, nmb in ((1, 1), (1, 4), (2, 3)):
            want = replay.deadlock_free(pl, Ks=(K,), n_mbs=(nmb,))
            assert R.rescclCheckDeadlock(text, f"fuse={fuse}", K, nmb) == want


def test_streaming_fusion_rejected_for_ring():
    text = R.rescclGenerateIr("ring", "allreduce", 4)
    js = R.rescclPlanIr(text, "fuse=1")
    assert js["plan"]["fused"] is False


def test_invalid_ir_rejected():
    bad = [
        "algo name=x coll=allreduce nranks=2 nchunks=2\nt 0 2 0 0 rrc\n",
        "algo name=x coll=allreduce nranks=2 nchunks=2\nt 0 0 0 0 rrc\n",
        "algo name=x coll=allreduce nranks=3 nchunks=3\nt 0 1 0 0 rrc\nt 2 1 0 0 rrc\n",
        "algo name=x coll=allgather nranks=3 nchunks=3\nt 1 2 0 0 recv\n",
        "algo name=x coll=allreduce nranks=2 nchunks=2\nt 0 1 0 0 add\n",
        "t 0 1 0 0 rrc\n",
        "algo name=x coll=allreduce nranks=2 nchunks=3\n",
    ]
    for b in bad:
        with pytest.raises(R.ResCCLError) as e:
            R.rescclPlanIr(b)
        assert e.value.code in (R.rescclInvalidUsage, R.rescclInvalidArgument)


def test_tb_budget_mapping():
    """a5: budget B >= T_min -> pair model, instances = floor(B/T_min); B < T_min -> port."""
    text = R.rescclGenerateIr("hm", "allreduce", 8, "g=4")
    js = R.rescclPlanIr(text, "tbbudget=8")
    assert js["linkmodel"] == "pair" and js["instances"] == 2 and js["ctas"] == [4] * 8
    js = R.rescclPlanIr(text, "tbbudget=2")
    assert js["linkmodel"] == "port" and js["instances"] == 2 and js["ctas"] == [1] * 8
    js = R.rescclPlanIr(text, "tbbudget=16")
    assert js["instances"] == 4


# ------------------------------------------------------------------ boundary

def _declared_symbols():
    hdr = open(os.path.join(os.path.dirname(__file__), "..", "include", "resccl.h")).read()
    return sorted(set(re.findall(r"\b(resccl[A-Z]\w+)\s*\(", hdr)))


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(R.LIB_PATH)
    syms = _declared_symbols()
    assert len(syms) >= 20
    for s in syms:
        assert hasattr(lib, s), s
    assert set(syms) == set(R.EXPORTS) | {"rescclCommInit"}


def test_error_strings_and_version():
    assert R.rescclGetErrorString(R.rescclTimeout).startswith("timeout")
    assert R.rescclGetVersion() == 1000


@pytest.mark.parametrize("name,coll,n,kw", [CASES[0], CASES[2], CASES[8], CASES[12], CASES[15], CASES[17],
                                            CASES[19]])
@pytest.mark.parametrize("dtype", [R.rescclFloat32, R.rescclBfloat16])
def test_generated_kernel_compiles_for_sm100a(name, coll, n, kw, dtype):
    """The generated kernel compiles with NVRTC for sm_100a (no GPU needed)."""
    text = _cpp_ir(name, coll, n, kw)
    assert R.rescclCompileIr(text, "instances=2", dtype, R.rescclSum) > 10000


@pytest.mark.parametrize("direct", [0, 1])
def test_multiprocess_rank_kernel_compiles(direct):
    """One rank's multi-process kernel (.sys scope); with direct=1 it carries the exit
    barrier that keeps peers' pulls/pushes inside the call (registered windows)."""
    text = _cpp_ir("ring", "allreduce", 4, {})
    assert R.rescclCompileIr(text, f"instances=2 sysrank=1 direct={direct}", R.rescclBfloat16, R.rescclSum) > 10000
    src = R.rescclCodegenIr(text, f"direct={direct}", 1, 2)
    assert "#define RESCCL_EXIT_BARRIER 0" in src  # CodegenIr leaves it to the runtime


def test_generated_code_has_no_interpreter():
    """§4.5: every primitive is a direct call with compile-time descriptor; no loop over
    a runtime program array."""
    text = _cpp_ir("ring", "allreduce", 4, {})
    src = R.rescclCodegenIr(text, "")
    assert src.count("rdev::run<") == 4 * 2 * 6  # 4 ranks x (send + recv) x 2(N-1) steps
    assert "switch (g / RESCCL_I)" in src


@pytest.mark.parametrize("name,coll,n,kw", CASES)
def test_round_robin_plan_matches_oracle(name, coll, n, kw):
    """RR baseline: C++ sched=rr == oracle hpds.round_robin."""
    g = _oracle_ir(name, coll, n, kw)
    js = R.rescclPlanIr(g.to_text(), "sched=rr")
    edges, _ = dag.build_dag(g)
    pr = hpds.round_robin(g, edges)
    tasks = [tuple(t) for t in js["plan"]["tasks"]]
    assert [[tasks[i] for i in pc] for pc in js["plan"]["Pr"]] == [[tuple(g.transfers[i]) for i in pc] for pc in pr]
    assert _norm_cpp(js) == _norm_oracle(lower.lower(g, "pair", Pr=pr))


@pytest.mark.parametrize("name,coll,n,kw", CASES)
@pytest.mark.parametrize("model", ["pair", "port"])
def test_direct_plan_matches_oracle(name, coll, n, kw, model):
    """Direct transport (R23): identical lowering (push/pull kinds, remote buffers, ack
    dependencies) in the C++ planner and the oracle, and the same deadlock verdicts."""
    g = _oracle_ir(name, coll, n, kw)
    js = R.rescclPlanIr(g.to_text(), f"linkmodel={model} direct=1")
    pl = lower.lower(g, model, direct=True)
    assert js["plan"]["direct"] is True and pl.direct
    assert _norm_cpp(js) == _norm_oracle(pl)
    for K, nmb in ((1, 1), (1, 3), (2, 16)):
        assert R.rescclCheckDeadlock(g.to_text(), f"linkmodel={model} direct=1", K, nmb) == \
            replay.deadlock_free(pl, Ks=(K,), n_mbs=(nmb,))


@pytest.mark.parametrize("name,coll,n,kw", CASES)
@pytest.mark.parametrize("model", ["pair", "port"])
def test_pushreduce_plan_matches_oracle(name, coll, n, kw, model):
    """Push-reduce variant of the direct transport (R31): rrc tasks keep the staged FIFO,
    recv tasks stay direct pushes; same lowering in the C++ planner and the oracle, and the
    same deadlock verdicts."""
    g = _oracle_ir(name, coll, n, kw)
    js = R.rescclPlanIr(g.to_text(), f"linkmodel={model} direct=1 pushreduce=1")
    pl = lower.lower(g, model, direct=True, pushreduce=True)
    assert js["plan"]["pushreduce"] is True and pl.pushreduce
    assert _norm_cpp(js) == _norm_oracle(pl)
    kinds = {p["kind"] for rp in js["plan"]["ranks"] for p in rp["prims"]}
    assert not kinds & {"psend", "prrc", "prrc_p", "prrc_d"}   # nothing is pulled
    for K, nmb in ((1, 1), (1, 3), (2, 16)):
        assert R.rescclCheckDeadlock(g.to_text(), f"linkmodel={model} direct=1 pushreduce=1", K, nmb) == \
            replay.deadlock_free(pl, Ks=(K,), n_mbs=(nmb,))
