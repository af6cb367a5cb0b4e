"""Pins of the CPU oracle against what the paper and the mathematics fix.

Each test names the passage (PAPER.md P:Lx-y) or closed form it checks.  None of
these tests touches the product path (C++ planner / CUDA kernels)."""
import itertools
import json
import os

import numpy as np
import pytest

import resccl_inputs as inp
from oracle import dag, definition, hpds, ir, lower, numerics, replay

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------------------- Fig. 5

def _fig5_ir():
    with open(os.path.join(GOLDEN, "fig5_ring_allgather_n4.txt")) as f:
        return ir.parse_text(f.read())


def test_fig5a_listing_matches_generator():
    """Fig. 5a listing written out by hand == ring_allgather(4)."""
    g = _fig5_ir()
    assert sorted(g.transfers) == sorted(ir.ring_allgather(4).transfers)


def test_fig5b_dag_has_12_nodes_and_chains():
    """Fig. 5b: 12 tasks v0-v11; only same-chunk, consecutive-step edges."""
    g = _fig5_ir()
    edges, _ = dag.build_dag(g)
    assert len(g.transfers) == 12
    assert len(edges) == 8
    for u, v in edges:
        tu, tv = g.transfers[u], g.transfers[v]
        assert tu.chunk == tv.chunk and tv.step == tu.step + 1 and tu.dst == tv.src


def test_fig5c_three_sub_pipelines_one_per_step():
    """Fig. 5c 'Sub Pipeline 0/1/2'."""
    g = _fig5_ir()
    edges, _ = dag.build_dag(g)
    Pr = hpds.hpds(g, edges, "pair")
    assert len(Pr) == 3
    for k, pc in enumerate(Pr):
        assert sorted(g.transfers[i].step for i in pc) == [k] * 4


def test_fig5e_rank0_uses_two_tbs():
    """Fig. 5e: rank 0 runs 'TB 0 / TB 1' (a send and a recv TB)."""
    pl = lower.lower(_fig5_ir(), "pair")
    assert pl.paper_tbs(0) == 2
    assert pl.send_groups[0] == [[(1, "send")]]
    assert pl.recv_groups[0] == [[(3, "recv")]]
    assert pl.ctas(0) == 1


# ----------------------------------------------------------------------------- Fig. 16

def _exec_fig16(n_nodes, g):
    with open(os.path.join(GOLDEN, "fig16_hm_allreduce.py.txt")) as f:
        src = f.read()
    src = src.replace("    nNodes = 4\n", f"    nNodes = {n_nodes}\n")
    src = src.replace("    nGpusperNode = 8\n", f"    nGpusperNode = {g}\n")
    out = []
    env = {"transfer": lambda s, d, st, c, op: out.append(ir.Transfer(s, d, st, c, op)),
           "rrc": "rrc", "recv": "recv"}
    exec(compile(src, "fig16", "exec"), env)
    env["ResCCLAlgo"]()
    return out


@pytest.mark.parametrize("n_nodes,g", [(2, 4), (2, 8), (4, 4), (4, 8)])
def test_fig16_listing_matches_generator(n_nodes, g):
    """The Fig. 16 program text, executed, == oracle.ir.hm_allreduce."""
    lst = _exec_fig16(n_nodes, g)
    assert sorted(lst) == sorted(ir.hm_allreduce(n_nodes, g).transfers)


@pytest.mark.parametrize("n_nodes,g", [(2, 4), (2, 8), (4, 4), (4, 8)])
def test_fig16_is_a_correct_allreduce(n_nodes, g):
    """Fig. 16 instantiated is conflict-free (I6), exactly-once (I1) and complete (I3)."""
    h = ir.hm_allreduce(n_nodes, g)
    dag.build_dag(h)
    replay.check_full_result(h, replay.symbolic(h))


def test_fig16_mutation_is_rejected():
    """One step changed in Fig. 16 must be caught by I1/I3/I6 (mutation test)."""
    h = ir.hm_allreduce(2, 4)
    caught = 0
    for k in range(0, len(h.transfers), 7):
        t = h.transfers[k]
        for delta in (-1, 1, 9):
            m = list(h.transfers)
            m[k] = t._replace(step=t.step + delta) if t.step + delta >= 0 else t._replace(chunk=(t.chunk + 1) % 8)
            mir = ir.IR(h.name, h.coll, h.nranks, h.nchunks, m)
            try:
                dag.build_dag(mir)
                replay.check_full_result(mir, replay.symbolic(mir))
                # semantics preserved?  then the value replay must still equal the definition
                xs = inp.all_inputs("int32", 3, 8, 64)
                out = replay.replay(lower.lower(mir), xs, "int32", 64, chunk_bytes=64)
                ref = definition.allreduce(xs, "int32")
                if all(np.array_equal(a, b) for a, b in zip(out, ref)):
                    continue
            except (dag.InvalidIR, AssertionError):
                pass
            caught += 1
    assert caught > 0
    # a mutation that changes a chunk id must always be caught
    m = list(h.transfers)
    m[0] = m[0]._replace(chunk=(m[0].chunk + 1) % 8)
    with pytest.raises((dag.InvalidIR, AssertionError)):
        mir = ir.IR(h.name, h.coll, h.nranks, h.nchunks, m)
        dag.build_dag(mir)
        replay.check_full_result(mir, replay.symbolic(mir))


# ----------------------------------------------------------------------------- Table 3

def test_table3_expert_tb_counts():
    """Table 3 ResCCL '# TB' for expert AR/AG = 8/16/8/16 on Topo1-4."""
    with open(os.path.join(GOLDEN, "table3_tb_counts.json")) as f:
        gold = json.load(f)
    for key, gen in (("expert_allreduce", ir.hm_allreduce), ("expert_allgather", ir.hm_allgather)):
        for topo, want in gold[key].items():
            nn, g = map(int, topo.split("x"))
            pl = lower.lower(gen(nn, g), "pair", fuse=False)
            for r in range(nn * g):
                assert pl.paper_tbs(r) == want, (key, topo, r)


def test_connection_based_allocation_is_upper_bound():
    """A8: connection-based #TB = |C| >= state-based |TB| (Eq. 7)."""
    for g in (ir.hm_allreduce(2, 4), ir.dbt_allreduce(8), ir.synth_allgather(8, 1, 3)):
        pl = lower.lower(g, "pair")
        for r in range(g.nranks):
            assert pl.paper_tbs(r) <= pl.n_connections[r]


# ----------------------------------------------------------------------------- Appendix A fixtures

def test_ring_ar2_plan_A1():
    """4 tasks, 2 edges, Pc0 = step-0 rrc, Pc1 = step-1 recv."""
    g = ir.ring_allreduce(2)
    edges, _ = dag.build_dag(g)
    assert len(g.transfers) == 4 and len(edges) == 2
    Pr = hpds.hpds(g, edges)
    assert [sorted(g.transfers[i] for i in pc) for pc in Pr] == [
        [(0, 1, 0, 0, "rrc"), (1, 0, 0, 1, "rrc")],
        [(0, 1, 1, 1, "recv"), (1, 0, 1, 0, "recv")]]


def test_hm_ar_2x4_plan_A3():
    """A.3: 112 tasks, 160 edges, 4 Pcs of 32/32/24/24 (steps 0-7, 0-7, 8-9, 8-9); no merging."""
    g = ir.hm_allreduce(2, 4)
    edges, _ = dag.build_dag(g)
    assert len(g.transfers) == 112 and len(edges) == 160
    Pr = hpds.hpds(g, edges)
    assert [len(p) for p in Pr] == [32, 32, 24, 24]
    assert {g.transfers[i].step for i in Pr[2]} | {g.transfers[i].step for i in Pr[3]} == {8, 9}
    pl = lower.lower(g, "pair", fuse=False)
    assert pl.n_connections[0] == 8 and pl.paper_tbs(0) == 8 and pl.ctas(0) == 4


def test_dbt8_parents_A4():
    (p1, r1), (p2, r2) = ir.dbt_trees(8)
    assert p1 == {1: 2, 2: 4, 3: 2, 4: 0, 5: 6, 6: 4, 7: 6} and r1 == 0
    assert p2 == {6: 5, 5: 3, 4: 5, 3: 7, 2: 1, 1: 3, 0: 1} and r2 == 7


@pytest.mark.parametrize("gen,want", [
    (lambda: ir.hm_allreduce(2, 4), 14), (lambda: ir.hm_allreduce(2, 8), 30),
    (lambda: ir.hm_allgather(2, 4), 7), (lambda: ir.dbt_allreduce(8), 28)])
def test_port_model_A5(gen, want):
    """A.5: port link model -> #Pc and 1 duplex CTA per rank."""
    g = gen()
    pl = lower.lower(g, "port")
    assert len(pl.Pr) == want
    assert all(pl.ctas(r) == 1 for r in range(g.nranks))


@pytest.mark.parametrize("n", [2, 3, 4, 5, 8, 16])
def test_ring_hpds_closed_form(n):
    """Ring under HPDS: Pc_k is exactly the set of step-k tasks."""
    for g in (ir.ring_allgather(n), ir.ring_reducescatter(n), ir.ring_allreduce(n)):
        edges, _ = dag.build_dag(g)
        Pr = hpds.hpds(g, edges)
        steps = max(t.step for t in g.transfers) + 1
        assert len(Pr) == steps
        for k, pc in enumerate(Pr):
            assert {g.transfers[i].step for i in pc} == {k} and len(pc) == n


@pytest.mark.parametrize("gen,coef", [
    (lambda n: ir.ring_allreduce(n), lambda n: 2 * (n - 1)),
    (lambda n: ir.ring_allgather(n), lambda n: (n - 1)),
    (lambda n: ir.ring_reducescatter(n), lambda n: (n - 1))])
def test_per_rank_egress_closed_form(gen, coef):
    """Per-rank NVLink egress in chunks: ring AR 2(N-1), AG/RS (N-1)."""
    for n in (2, 4, 8):
        g = gen(n)
        for r in range(n):
            assert sum(1 for t in g.transfers if t.src == r) == coef(n)


def test_hm_ar_2x4_egress_equals_ring():
    """HM-AR 2x4 per-rank egress = 14 chunks = ring AR's 2(N-1) (derived)."""
    g = ir.hm_allreduce(2, 4)
    assert all(sum(1 for t in g.transfers if t.src == r) == 14 for r in range(8))


def test_dbt8_busiest_rank_sends_2S():
    """A.4: DBT-8 per-rank egress: ranks 0,7 send N/... = 1.0 S, ranks 1-6 send 2.0 S."""
    g = ir.dbt_allreduce(8)
    eg = [sum(1 for t in g.transfers if t.src == r) for r in range(8)]
    assert eg == [8, 16, 16, 16, 16, 16, 16, 8]


# ----------------------------------------------------------------------------- numerics

def test_bf16_rne_ties_and_known_values():
    """RNE to bfloat16 on hand-computed values (IEEE 754 roundTiesToEven)."""
    f = np.array([1.0, 1.00390625, 1.01171875, 1.0078125 + 2 ** -20, -2.5, 3.0e38], dtype=np.float32)
    # 1+2^-8 is a tie -> even (1.0); 1+3*2^-8 tie -> 1+2^-6 (even mantissa 2);
    got = numerics.f32_to_bf16_rne(f)
    assert list(got[:3]) == [0x3F80, 0x3F80, 0x3F82]
    assert got[3] == 0x3F81          # above the tie rounds up... 1+2^-7 exactly representable
    assert got[4] == 0xC020
    assert numerics.bf16_to_f32(np.array([0x3F80], np.uint16))[0] == 1.0


def test_f64_to_bf16_vectorised_matches_scalar():
    rng = np.random.default_rng(0)
    d = rng.standard_normal(5000) * np.exp(rng.uniform(-20, 20, 5000))
    a = numerics.f64_to_dtype_rne(d, "bfloat16")
    b = np.array([numerics.f64_to_bf16_scalar(float(x)) for x in d], dtype=np.uint16)
    assert np.array_equal(a, b)


@pytest.mark.parametrize("dtype", ["bfloat16", "float16"])
def test_R8_fp32_then_round_is_correctly_rounded_add(dtype):
    """Reading R8: (a+b) in binary32 then RNE == correctly rounded 16-bit add
    (24 >= 2p+2 for p = 8, 11).  Checked against binary64 + single rounding."""
    rng = np.random.default_rng(1)
    for scale in (1.0, 1e-3, 1e3):
        f = (rng.standard_normal(200000) * scale).astype(np.float32)
        g = (rng.standard_normal(200000) * scale).astype(np.float32)
        a = numerics.from_f32(f, dtype)
        b = numerics.from_f32(g, dtype)
        got = numerics.combine(a, b, dtype)
        exact = numerics.to_f32(a, dtype).astype(np.float64) + numerics.to_f32(b, dtype).astype(np.float64)
        want = numerics.f64_to_dtype_rne(exact, dtype)
        assert np.array_equal(got.view(np.uint16), want.view(np.uint16))


def test_int32_sum_wraps():
    a = np.array([2 ** 31 - 1, -2 ** 31], dtype=np.int32)
    b = np.array([1, -1], dtype=np.int32)
    assert list(numerics.combine(a, b, "int32")) == [-2 ** 31, 2 ** 31 - 1]


# ----------------------------------------------------------------------------- definition

@pytest.mark.parametrize("dtype", ["int32", "float32", "float16", "bfloat16"])
def test_definition_exact_inputs_equal_python_integer_sum(dtype):
    """Exact mode: integers in [-4,4]; sums of <=8 are exact in every dtype, so the
    definition equals the integer sum computed with Python ints."""
    xs = inp.all_inputs(dtype, 5, 8, 333, "exact")
    out = definition.reduce_all(xs, dtype)
    ints = [numerics.to_f32(x, dtype).astype(np.int64) if dtype != "int32" else x.astype(np.int64)
            for x in xs]
    want = [sum(int(v[i]) for v in ints) for i in range(333)]
    got = numerics.to_f32(out, dtype) if dtype != "int32" else out
    assert [int(v) for v in got] == want


def test_definition_allgather_reducescatter_layout():
    xs = [np.arange(6, dtype=np.int32) + 100 * k for k in range(3)]
    ag = definition.allgather(xs)
    assert list(ag[1]) == list(range(6)) + list(range(100, 106)) + list(range(200, 206))
    rs = definition.reducescatter(xs, "int32")
    assert list(rs[2]) == [3 * 4 + 300, 3 * 5 + 300]


def test_definition_int32_wraparound():
    xs = inp.all_inputs("int32", 0, 8, 1000, "wrap")
    out = definition.reduce_all(xs, "int32")
    want = [((sum(int(x[i]) for x in xs) + 2 ** 31) % 2 ** 32) - 2 ** 31 for i in range(1000)]
    assert [int(v) for v in out] == want


# ----------------------------------------------------------------------------- replay

ALGOS = [
    ("ring", "allreduce", 2), ("ring", "allreduce", 3), ("ring", "allreduce", 8),
    ("ring", "allgather", 4), ("ring", "reducescatter", 5), ("dbt", "allreduce", 4),
    ("dbt", "allreduce", 8), ("dbt", "allreduce", 6), ("hm", "allreduce", 8),
    ("hm", "allgather", 8), ("synth", "allgather", 8), ("synth", "reducescatter", 8),
]


def _gen(name, coll, n):
    if name == "synth":
        return ir.generate(name, coll, n, seed=2, fanout=3)
    return ir.generate(name, coll, n)


def _defn(coll, xs, dtype, op="sum"):
    if coll == "allreduce":
        return definition.allreduce(xs, dtype, op)
    if coll == "allgather":
        return definition.allgather(xs)
    return definition.reducescatter(xs, dtype, op)


@pytest.mark.parametrize("name,coll,n", ALGOS)
@pytest.mark.parametrize("model", ["pair", "port"])
def test_replay_int32_equals_definition(name, coll, n, model):
    """int32 (any schedule) must equal the definition bit for bit (c5), incl. ragged tails."""
    g = _gen(name, coll, n)
    pl = lower.lower(g, model)
    for cnt in (1, 1000, 4097):
        m = cnt * n if coll == "reducescatter" else cnt
        xs = inp.all_inputs("int32", 7, n, m)
        for inplace in (False, True):
            out = replay.replay(pl, xs, "int32", cnt, chunk_bytes=1024, instances=3, K=2,
                                inplace=inplace)
            for a, b in zip(out, _defn(coll, xs, "int32")):
                assert np.array_equal(a, b)


@pytest.mark.parametrize("name,coll,n", ALGOS)
@pytest.mark.parametrize("dtype", ["float32", "float16", "bfloat16"])
def test_replay_exact_inputs_equal_definition(name, coll, n, dtype):
    """Exactly-representable inputs: every order gives the same bits (c5)."""
    g = _gen(name, coll, n)
    pl = lower.lower(g)
    cnt = 777
    m = cnt * n if coll == "reducescatter" else cnt
    xs = inp.all_inputs(dtype, 11, n, m, "exact")
    out = replay.replay(pl, xs, dtype, cnt, chunk_bytes=512, instances=2, K=1)
    for a, b in zip(out, _defn(coll, xs, dtype)):
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))


@pytest.mark.parametrize("name,coll,n", [a for a in ALGOS if a[1] != "allgather"])
@pytest.mark.parametrize("dtype,rtol", [("float32", 1e-5), ("bfloat16", 2e-2), ("float16", 2e-2)])
def test_replay_within_tolerance_of_naive(name, coll, n, dtype, rtol):
    """north_star tolerance: |g - ref| <= rtol * sum_k |x_k| (cancellation-safe)."""
    g = _gen(name, coll, n)
    pl = lower.lower(g)
    cnt = 2000
    m = cnt * n if coll == "reducescatter" else cnt
    xs = inp.all_inputs(dtype, 1, n, m)
    out = replay.replay(pl, xs, dtype, cnt, chunk_bytes=2048, instances=2, K=2)
    ref = _defn(coll, xs, dtype)
    den = definition.abs_sum(xs, dtype)
    for r, (a, b) in enumerate(zip(out, ref)):
        d = den if coll == "allreduce" else den[r * cnt:(r + 1) * cnt]
        diff = np.abs(numerics.to_f32(a, dtype).astype(np.float64) - numerics.to_f32(b, dtype).astype(np.float64))
        assert np.all(diff <= rtol * d + 1e-30)


@pytest.mark.parametrize("n", [2, 3, 4, 8])
def test_ring_allreduce_fp32_closed_form_order(n):
    """Ring AR (R10) reduces chunk c in ring order starting at rank c:
    v = x_{c+N-1} + (... + (x_{c+1} + x_c)) in binary32 (local + incoming)."""
    g = ir.ring_allreduce(n)
    pl = lower.lower(g)
    cnt = 64 * n * 3
    xs = inp.all_inputs("float32", 4, n, cnt)
    out = replay.replay(pl, xs, "float32", cnt, chunk_bytes=256, instances=1, K=2)
    C = cnt // n
    for c in range(n):
        acc = xs[c][c * C:(c + 1) * C].astype(np.float32)
        for k in range(1, n):
            acc = (xs[(c + k) % n][c * C:(c + 1) * C] + acc).astype(np.float32)
        for r in range(n):
            assert np.array_equal(out[r][c * C:(c + 1) * C], acc)


def test_replay_max_min_order_free():
    for name, coll, n in [("ring", "allreduce", 4), ("dbt", "allreduce", 8), ("ring", "reducescatter", 4)]:
        g = _gen(name, coll, n)
        pl = lower.lower(g)
        for dtype in ("float32", "bfloat16", "int32"):
            for op in ("max", "min"):
                cnt = 300
                m = cnt * n if coll == "reducescatter" else cnt
                xs = inp.all_inputs(dtype, 9, n, m)
                out = replay.replay(pl, xs, dtype, cnt, op=op, chunk_bytes=256)
                for a, b in zip(out, _defn(coll, xs, dtype, op)):
                    assert np.array_equal(a.view(np.uint8), b.view(np.uint8))


@pytest.mark.parametrize("name,coll,n", ALGOS)
def test_all_interleavings_same_bytes(name, coll, n):
    """I2 (brute force): random interleavings give byte-identical results."""
    g = _gen(name, coll, n)
    pl = lower.lower(g)
    cnt = 200
    m = cnt * n if coll == "reducescatter" else cnt
    xs = inp.all_inputs("float32", 2, n, m)
    base = replay.replay(pl, xs, "float32", cnt, chunk_bytes=64, instances=2, K=1)
    for seed in range(4):
        o = replay.replay(pl, xs, "float32", cnt, chunk_bytes=64, instances=2, K=1,
                          sched="random", seed=seed)
        for a, b in zip(base, o):
            assert np.array_equal(a.view(np.uint8), b.view(np.uint8))


@pytest.mark.parametrize("name,coll,n", ALGOS)
@pytest.mark.parametrize("model", ["pair", "port"])
def test_happens_before_no_races(name, coll, n, model):
    """I2 (proof): every conflicting access pair is ordered by happens-before."""
    pl = lower.lower(_gen(name, coll, n), model)
    for n_mb, K in ((1, 1), (2, 1), (3, 2)):
        for inplace in (False, True):
            assert replay.happens_before_races(pl, n_mb=n_mb, instances=1, K=K, inplace=inplace) == []


def test_exhaustive_interleavings_tiny():
    """I2 by brute force: every interleaving of ring AR N=2 and N=3 with n_mb=2, K=1."""
    for n in (2, 3):
        pl = lower.lower(ir.ring_allreduce(n))
        g = replay.Geometry("allreduce", n, 128 * n, 4, 256, 1)
        assert g.n_mb == 2
        xs = inp.all_inputs("float32", 0, n, 128 * n)
        results = set()
        states = [0]

        def explore(seq_seed_budget):
            pass

        # enumerate schedules by DFS over enabled processes
        import copy
        sim0 = replay._Sim(pl, g.n_mb, 1, 1)
        bufs0 = replay.make_buffers(pl, xs, "float32", 128 * n)

        def action_factory(bufs):
            def action(p, r, j, inst, incoming):
                lo, hi = g.slice(p.chunk, j, inst)
                if p.recv_task is None:
                    o = g.chunk_off(p.src_buf, p.chunk)
                    return bufs[r][p.src_buf][o + lo:o + hi].copy()
                v = numerics.combine(bufs[r][p.src_buf][g.chunk_off(p.src_buf, p.chunk) + lo:
                                                       g.chunk_off(p.src_buf, p.chunk) + hi],
                                     incoming, "float32") if p.reduce else incoming
                if p.store:
                    o = g.chunk_off(p.dst_buf, p.chunk)
                    bufs[r][p.dst_buf][o + lo:o + hi] = v
                return v.copy()
            return action

        def dfs(sim, bufs, depth):
            if sim.finished():
                results.add(b"".join(b["recv"].tobytes() for b in bufs))
                states[0] += 1
                return
            en = [k for k, pr in enumerate(sim.procs) if sim.enabled(pr)]
            assert en, "deadlock"
            for k in en:
                s2 = copy.deepcopy(sim)
                b2 = copy.deepcopy(bufs)
                s2.fire(s2.procs[k], action_factory(b2))
                dfs(s2, b2, depth + 1)
                if states[0] > 3000:
                    return

        dfs(sim0, bufs0, 0)
        assert states[0] > 1 and len(results) == 1


@pytest.mark.parametrize("name,coll,n", ALGOS)
def test_plan_well_formed_and_deadlock_free(name, coll, n):
    """I4 + I5 for both link models."""
    for model in ("pair", "port"):
        pl = lower.lower(_gen(name, coll, n), model)
        replay.check_plan(pl)
        assert replay.deadlock_free(pl, Ks=(1, 2), n_mbs=(1, 2, 3, 16))


def test_streaming_fusion_of_ring_deadlocks_and_is_rejected():
    """Task-level execution + recvReduceSend streaming on the ring forms a cyclic wait
    for n_mb > K (derived); the lowering must fall back to unfused primitives."""
    pl = lower.lower(ir.ring_allreduce(4), fuse=True)
    assert not pl.fused
    kinds = {p.kind for r in pl.prims for p in pl.prims[r]}
    assert kinds == {"send", "rrc", "recv"}


def test_hm_fusion_kept():
    pl = lower.lower(ir.hm_allreduce(2, 4), fuse=True)
    assert pl.fused
    kinds = {p.kind for r in pl.prims for p in pl.prims[r]}
    assert kinds & {"rrs", "rcs", "rrcs"}


def test_round_robin_baseline_valid():
    """RR baseline yields a valid plan too (I5)."""
    for g in (ir.hm_allreduce(2, 4), ir.synth_allgather(8, 0, 2)):
        edges, _ = dag.build_dag(g)
        Pr = hpds.round_robin(g, edges)
        pl = lower.lower(g, Pr=Pr)
        replay.check_plan(pl)


def test_invalid_ir_rejected():
    """I6: out-of-range ranks, self transfers, same-step conflicts, undefined reads."""
    bad = [
        ir.IR("x", "allreduce", 2, 2, [ir.Transfer(0, 2, 0, 0, "rrc")]),
        ir.IR("x", "allreduce", 2, 2, [ir.Transfer(0, 0, 0, 0, "rrc")]),
        ir.IR("x", "allreduce", 3, 3, [ir.Transfer(0, 1, 0, 0, "rrc"), ir.Transfer(2, 1, 0, 0, "rrc")]),
        ir.IR("x", "allgather", 3, 3, [ir.Transfer(1, 2, 0, 0, "recv")]),
    ]
    for b in bad:
        with pytest.raises(dag.InvalidIR):
            dag.build_dag(b)
            dag.check_defined_reads(b)


def test_text_roundtrip():
    for g in (ir.hm_allreduce(2, 4), ir.synth_reducescatter(8, 3, 2)):
        assert ir.parse_text(g.to_text()) == g


# ----------------------------------------------------------------------------- direct transport (R23)

@pytest.mark.parametrize("name,coll,n", ALGOS)
def test_direct_transport_replay_and_races(name, coll, n):
    """Direct push/pull semantics give the definition (int32), the staged mode's bytes
    (fp32), no happens-before races and no deadlock."""
    g = _gen(name, coll, n)
    pd = lower.lower(g, "pair", direct=True)
    ps = lower.lower(g, "pair")
    cnt = 500
    m = cnt * n if coll == "reducescatter" else cnt
    xs = inp.all_inputs("int32", 4, n, m)
    out = replay.replay(pd, xs, "int32", cnt, chunk_bytes=256, instances=2, K=1)
    for a, b in zip(out, _defn(coll, xs, "int32")):
        assert np.array_equal(a, b)
    xf = inp.all_inputs("float32", 4, n, m)
    od = replay.replay(pd, xf, "float32", cnt, chunk_bytes=256, instances=2, K=1, sched="random", seed=1)
    os_ = replay.replay(ps, xf, "float32", cnt, chunk_bytes=256, instances=2, K=1)
    for a, b in zip(od, os_):
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))
    for n_mb, K in ((1, 1), (2, 1), (3, 2)):
        for inplace in (False, True):
            assert replay.happens_before_races(pd, n_mb=n_mb, instances=1, K=K, inplace=inplace) == []
    assert replay.deadlock_free(pd, Ks=(1,), n_mbs=(1, 2, 3, 16))


def test_direct_race_checker_catches_missing_ack_dependency():
    """Mutation: dropping the pull-send acknowledgement dependencies lets a later write
    of the sender's location race with the peer's pull -- the I2 checker must see it."""
    # rank 1 pulls <0,0> (rrc, step 0); rank 2 then overwrites <0,0> (recv, step 1) with a
    # value that does not depend on that read: only the ack dependency orders them
    # (in-place: the pulled send-buffer copy and the pushed receive-buffer copy alias)
    g = ir.IR("x", "allreduce", 3, 3, [ir.Transfer(0, 1, 0, 0, "rrc"), ir.Transfer(2, 0, 1, 0, "recv")])
    pd = lower.lower(g, "pair", direct=True)
    assert replay.happens_before_races(pd, n_mb=2, instances=1, K=1, inplace=True) == []
    assert any(p.ack_deps for r in pd.prims for p in pd.prims[r])
    for r in pd.prims:
        for p in pd.prims[r]:
            p.ack_deps = []
    assert replay.happens_before_races(pd, n_mb=2, instances=1, K=1, inplace=True) != []


# ----------------------------------------------------------------------------- flag rings (R26)

@pytest.mark.parametrize("name,coll,n,kw", [("ring", "allreduce", 8, {}),
                                            ("synth", "reducescatter", 8, {"seed": 0, "fanout": 2}),
                                            ("dbt", "allreduce", 8, {}), ("hm", "allreduce", 8, {"g": 4})])
def test_flag_rings_per_sending_lane(name, coll, n, kw):
    """R26: with the device's flag encoding (slot pos % K overwritten with pos + 1, the
    receiver tests slot >= pos + 1), one ring per link is wrong under the direct
    transport -- a pull-send posts without a credit wait, and a link fed by two lanes
    (a fused forward beside a plain send) can post out of order: the receiver sees a
    position early or loses one.  One ring per (link, sending lane) makes the device
    test agree with the ideal "posted" everywhere, for both transports."""
    g = ir.generate(name, coll, n, **kw)
    for direct in (False, True):
        p = lower.lower(g, "pair", direct=direct)
        link_bad = 0
        for K in (1, 2):
            for n_mb in (1, 2, 3):
                for sched, seed in (("rr", 0), ("random", 1), ("random", 2)):
                    s = replay._Sim(p, n_mb, 1, K, rings="lane")
                    s.run(sched, seed)
                    assert s.hazards == [], (direct, K, n_mb, sched, s.hazards[:3])
                    s = replay._Sim(p, n_mb, 1, K, rings="link")
                    s.run(sched, seed)
                    link_bad += bool(s.hazards)
                    if not direct:
                        assert s.hazards == []  # staged: the FIFO credit orders every post
        if direct and name in ("ring", "synth"):
            assert link_bad > 0  # the per-link encoding is observably broken here
