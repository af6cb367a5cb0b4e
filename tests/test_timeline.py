"""f2: the wall-clock timeline under the alpha-beta cost model with Eq. 1 contention
(C++ rescclSimulateTimeline vs the oracle's oracle/timeline.py), pinned to closed
forms of the paper's equations.  No GPU needed."""
import math

import pytest

import paper_conf_sigcomm_liuhlgcwz025_b200 as R
from oracle import dag, hpds, ir as oir, lower, replay, timeline

ALPHA, BETA, GAMMA = 2e-6, 1 / 900e9, 3e-6


def _cpp(g, opts, count, elt=2, alpha=ALPHA, beta=BETA, gamma=GAMMA):
    return R.rescclSimulateTimeline(g.to_text(), opts, count=count, elt=elt, alpha=alpha, beta=beta, gamma=gamma)


def _geom(g, count, elt, chunk_bytes, instances):
    geo = replay.Geometry(g.coll, g.nranks, count, elt, chunk_bytes, instances)
    return geo.n_mb, geo.Mi * elt


CASES = [("ring", "allreduce", 8, {}), ("ring", "allgather", 4, {}), ("dbt", "allreduce", 8, {}),
         ("hm", "allreduce", 8, {"g": 4}), ("hm", "allgather", 8, {"g": 4}),
         ("synth", "reducescatter", 8, {"seed": 1, "fanout": 3}), ("synth", "allgather", 8, {"seed": 0, "fanout": 2})]


@pytest.mark.parametrize("name,coll,n,kw", CASES)
@pytest.mark.parametrize("model,direct,sched,inst", [("pair", 0, "hpds", 1), ("pair", 1, "hpds", 2),
                                                      ("port", 0, "hpds", 1), ("pair", 0, "rr", 2)])
def test_timeline_matches_oracle(name, coll, n, kw, model, direct, sched, inst):
    g = oir.generate(name, coll, n, **kw)
    count, elt, cb = 3 << 20, 2, 1 << 20
    opts = f"linkmodel={model} direct={direct} sched={sched} instances={inst} chunkbytes={cb} fifodepth=2"
    js = _cpp(g, opts, count, elt)
    n_mb, c = _geom(g, count, elt, cb, inst)
    assert (js["n_mb"], js["c"], js["K"], js["instances"]) == (n_mb, c, 2, inst)
    edges, _ = dag.build_dag(g)
    pr = hpds.round_robin(g, edges, model) if sched == "rr" else None
    pl = lower.lower(g, model, Pr=pr, direct=bool(direct))
    o = timeline.timeline(pl, n_mb, 2, inst, c, ALPHA, BETA, GAMMA)
    assert math.isclose(js["makespan_s"], o["makespan_s"], rel_tol=1e-9)
    assert math.isclose(js["comm_time"], o["comm_time"], rel_tol=1e-9)
    assert math.isclose(js["max_idle"], o["max_idle"], rel_tol=1e-9, abs_tol=1e-12)
    assert js["max_z"] == o["max_z"]
    for r in range(n):
        assert js["ranks"][r]["merged_send"] == o["merged"][(r, "send")]
        assert js["ranks"][r]["merged_recv"] == o["merged"][(r, "recv")]


@pytest.mark.parametrize("n", [2, 4, 8])
@pytest.mark.parametrize("n_mb", [1, 2, 7])
def test_ring_allgather_closed_form(n, n_mb):
    """Ring AG, one instance, no contention: each send lane is busy back to back.
    For n_mb >= 2 (and alpha < tau) T = (N-1) n_mb tau + alpha, with tau = alpha + c beta
    (the last receive drains in alpha).  For n_mb = 1 every hop waits for the previous
    drain: T = (N-1)(tau + alpha)."""
    g = oir.ring_allgather(n)
    pl = lower.lower(g)
    c = 1 << 20
    tau = ALPHA + c * BETA
    o = timeline.timeline(pl, n_mb, 4, 1, c, ALPHA, BETA, GAMMA)
    want = (n - 1) * n_mb * tau + ALPHA if n_mb >= 2 else (n - 1) * (tau + ALPHA)
    assert math.isclose(o["makespan_s"], want, rel_tol=1e-12)
    assert o["max_z"] == 1


@pytest.mark.parametrize("z", [1, 2, 3, 5])
@pytest.mark.parametrize("n_mb", [1, 4])
def test_eq1_contention(z, n_mb):
    """Eq. 1: z identical tasks of n invocations sharing one link end at
    n z (alpha + c beta) + L(z) gamma, L(z) = z - 1.  Ring AG N=2 with z instances puts
    z send lanes on link (0,1); the last receive adds alpha (n_mb = 1 also waits for
    nothing else)."""
    g = oir.ring_allgather(2)
    pl = lower.lower(g)
    c = 1 << 20
    tau = ALPHA + c * BETA
    o = timeline.timeline(pl, n_mb, 4, z, c, ALPHA, BETA, GAMMA)
    assert math.isclose(o["makespan_s"], n_mb * z * tau + (z - 1) * GAMMA + ALPHA, rel_tol=1e-12)
    assert o["max_z"] == z
    js = _cpp(g, f"instances={z} chunkbytes={(c * z)}", (c * z * n_mb) // 2)
    assert (js["n_mb"], js["c"]) == (n_mb, c)
    assert math.isclose(js["makespan_s"], o["makespan_s"], rel_tol=1e-12)


def test_port_model_serialises_a_rank():
    """Port model (R2): the planner gives each rank one duplex CTA, so its sends to the
    three local peers of HM 2x4 AllGather run one after another on the egress port:
    no contention (z = 1), and a longer makespan than the pair model's parallel lanes."""
    g = oir.hm_allgather(2, 4)
    o_pair = timeline.timeline(lower.lower(g, "pair"), 2, 4, 1, 1 << 20, ALPHA, BETA, 0.0)
    o_port = timeline.timeline(lower.lower(g, "port"), 2, 4, 1, 1 << 20, ALPHA, BETA, 0.0)
    assert o_pair["max_z"] == 1 and o_port["max_z"] == 1
    assert o_port["makespan_s"] > 2 * o_pair["makespan_s"]


def test_hpds_beats_round_robin_on_dbt():
    """Fig. 10b's claim as a property of the model: HPDS's sub-pipelines finish DBT-8
    AllReduce no later than round-robin's."""
    g = oir.dbt_allreduce(8)
    edges, _ = dag.build_dag(g)
    o_h = timeline.timeline(lower.lower(g), 8, 2, 1, 1 << 20, ALPHA, BETA, GAMMA)
    o_r = timeline.timeline(lower.lower(g, Pr=hpds.round_robin(g, edges)), 8, 2, 1, 1 << 20, ALPHA, BETA, GAMMA)
    assert o_h["makespan_s"] < o_r["makespan_s"]


def test_wall_clock_merge_is_never_below_the_clique_bound():
    """Eq. 7 on active_l(t): merged lanes >= the most connections active at one instant,
    and ring's two connections per rank stay separate."""
    g = oir.ring_allreduce(8)
    o = timeline.timeline(lower.lower(g), 4, 2, 1, 1 << 20, ALPHA, BETA, GAMMA)
    for r in range(8):
        assert o["merged"][(r, "send")] == 1 and o["merged"][(r, "recv")] == 1
    g = oir.hm_allreduce(2, 4)
    o = timeline.timeline(lower.lower(g), 4, 2, 1, 1 << 20, ALPHA, BETA, GAMMA)
    for r in range(8):
        for d in ("send", "recv"):
            ivs = [iv for (rr, _, dd), iv in o["active"].items() if rr == r and dd == d]
            pts = sorted({a for iv in ivs for a, _ in iv})
            clique = max(sum(any(a <= p < b for a, b in iv) for iv in ivs) for p in pts)
            assert o["merged"][(r, d)] >= clique
