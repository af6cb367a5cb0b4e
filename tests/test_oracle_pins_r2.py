"""Round-2 pins of two oracle functions that were pinned only by the product before.

* ``replay.dataflow_values`` (step-order evaluation of the IR, the expectation of every
  full-size GPU parity test) is checked against ``replay.replay`` (the blocking FIFO
  simulator of the lowered plan) byte for byte: both must realise the same association
  order (reading R8) although one walks IR steps and the other lanes, micro-batches and
  instances.  Every algorithm of the pin suite, four dtypes, in and out of place,
  ragged counts.
* ``hpds.round_robin`` (the RR baseline) is checked against Pc lists
  derived by hand from that passage (``tests/golden/rr_pc_lists.txt``), and the C++
  planner's ``sched=rr`` against the same golden lists.
"""
import os
import re

import numpy as np
import pytest

import resccl_inputs as inp
from oracle import dag, hpds, ir as oir, lower, replay

GOLD = os.path.join(os.path.dirname(__file__), "golden")

ALGOS = [
    ("ring", "allreduce", 2, {}), ("ring", "allreduce", 3, {}), ("ring", "allreduce", 8, {}),
    ("ring", "allgather", 4, {}), ("ring", "reducescatter", 5, {}),
    ("dbt", "allreduce", 8, {}), ("dbt", "allreduce", 5, {}),
    ("hm", "allreduce", 8, {"g": 4}), ("hm", "allgather", 8, {"g": 4}),
    ("synth", "allgather", 6, {"seed": 1, "fanout": 2}),
    ("synth", "reducescatter", 6, {"seed": 2, "fanout": 3}),
    ("synth", "reducescatter", 8, {"seed": 0, "fanout": 2}),
]


def _chunk_inputs(coll, xs, geo, n):
    """Split every rank's input into the IR's chunks (reading R6)."""
    rows = []
    for r in range(n):
        row = []
        for c in range(n):
            if coll == "allgather":
                row.append(xs[r].copy() if r == c else None)
            else:
                o = geo.chunk_off("send", c)
                row.append(xs[r][o:o + geo.chunk_len[c]].copy())
        rows.append(row)
    return rows


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
@pytest.mark.parametrize("dtype", ["int32", "float32", "float16", "bfloat16"])
@pytest.mark.parametrize("inplace", [False, True])
def test_dataflow_values_equals_replay(name, coll, n, kw, dtype, inplace):
    g = oir.generate(name, coll, n, **kw)
    pl = lower.lower(g)
    for count, cb, inst in ((1, 256, 1), (4097, 1024, 3), (3 * 1024 + 5, 2048, 2)):
        xs = inp.all_inputs(dtype, 7, n, count * (n if coll == "reducescatter" else 1))
        geo = replay.Geometry(coll, n, count, replay.ELT[dtype], cb, inst)
        got = replay.replay(pl, xs, dtype, count, chunk_bytes=cb, instances=inst, K=2, inplace=inplace)
        exp = replay.dataflow_values(g, _chunk_inputs(coll, xs, geo, n), dtype)
        for r in range(n):
            for c in range(n):
                if coll == "reducescatter" and c != r:
                    continue
                o = geo.chunk_off("recv", c)
                ln = geo.chunk_len[c]
                a = np.ascontiguousarray(got[r][o:o + ln]).view(np.uint8)
                b = np.ascontiguousarray(exp[r][c]).view(np.uint8)
                assert np.array_equal(a, b), (count, r, c)


def test_dataflow_values_detects_a_wrong_step_order():
    """A plausible bug -- applying ring AllReduce's transfers in the wrong order (the
    AllGather half first) -- must change the result, so the test above can fail."""
    g = oir.generate("ring", "allreduce", 4)
    xs = inp.all_inputs("float32", 3, 4, 1024)
    geo = replay.Geometry("allreduce", 4, 1024, 4, 1 << 20, 1)
    ci = _chunk_inputs("allreduce", xs, geo, 4)
    good = replay.dataflow_values(g, ci, "float32")
    bad_ir = oir.IR(g.name, g.coll, g.nranks, g.nchunks, [oir.Transfer(t.src, t.dst, (t.step + 3) % 6, t.chunk, t.op)
                                                          for t in g.transfers])
    bad = replay.dataflow_values(bad_ir, ci, "float32")
    assert any(not np.array_equal(good[r][c], bad[r][c]) for r in range(4) for c in range(4))


# ---------------------------------------------------------------- round robin, hand-derived

def _gold_rr():
    names = {}
    for line in open(os.path.join(GOLD, "rr_pc_lists.txt")):
        m = re.match(r"#\s+(tree 1|tree 2):\s+(.*)", line)
        if m:
            names[m.group(1)] = dict(re.findall(r"(\w+) \((\d+,\d+,\d+)\)", m.group(2)))
            key = m.group(1)
        elif line.startswith("#           ") and names:
            names[key].update(re.findall(r"(\w+) \((\d+,\d+,\d+)\)", line))
    lists = {}
    for line in open(os.path.join(GOLD, "rr_pc_lists.txt")):
        m = re.match(r"(\w+) Pc(\d+): (.*)", line)
        if m:
            lists.setdefault(m.group(1), {}).setdefault(int(m.group(2)), []).extend(m.group(3).split())
    return names, lists


def _expand(algo, tok, names):
    nm, c = tok.split("@")
    c = int(c)
    if algo == "ring4":
        s = int(nm[1:])
        base = c if s < 3 else c + 3
        src = (base + (s if s < 3 else s - 3)) % 4
        return (c, s, src, (src + 1) % 4)
    tree = "tree 1" if c < 4 else "tree 2"
    step, src, dst = (int(v) for v in names[tree][nm].split(","))
    return (c, step, src, dst)


@pytest.mark.parametrize("algo,gen", [("ring4", ("ring", 4)), ("dbt8", ("dbt", 8))])
def test_round_robin_equals_hand_derived_golden(algo, gen):
    names, lists = _gold_rr()
    want = [[_expand(algo, tok, names) for tok in lists[algo][k]] for k in sorted(lists[algo])]
    g = oir.generate(gen[0], "allreduce", gen[1])
    edges, _ = dag.build_dag(g)
    pr = hpds.round_robin(g, edges, "pair")
    ts = g.transfers
    got = [[(ts[i].chunk, ts[i].step, ts[i].src, ts[i].dst) for i in pc] for pc in pr]
    assert got == want
    assert sum(len(p) for p in want) == len(ts)


@pytest.mark.parametrize("algo,gen", [("ring4", ("ring", 4)), ("dbt8", ("dbt", 8))])
def test_cpp_round_robin_equals_hand_derived_golden(algo, gen):
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    names, lists = _gold_rr()
    want = [[_expand(algo, tok, names) for tok in lists[algo][k]] for k in sorted(lists[algo])]
    g = oir.generate(gen[0], "allreduce", gen[1])
    js = R.rescclPlanIr(g.to_text(), "sched=rr")
    tasks = js["plan"]["tasks"]
    got = [[(tasks[i][3], tasks[i][2], tasks[i][0], tasks[i][1]) for i in pc] for pc in js["plan"]["Pr"]]
    assert got == want


def test_round_robin_differs_from_hpds_on_dbt8():
    """The pin distinguishes the two schedulers: HPDS (priorities) interleaves all eight
    chunks into 4 large sub-pipelines, RR walks whole trees."""
    g = oir.generate("dbt", "allreduce", 8)
    edges, _ = dag.build_dag(g)
    assert [len(p) for p in hpds.round_robin(g, edges)] == [24, 16, 16, 16, 4, 12, 12, 12]
    assert [len(p) for p in hpds.hpds(g, edges)] == [24, 24, 24, 24, 4, 4, 4, 4]


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
def test_pushreduce_replay_definition_races_deadlock(name, coll, n, kw):
    """R31 plans: int32 results equal the definition, the happens-before check finds no
    race (a staged slot and a direct push share one link's credit counter and flag ring),
    and the blocking model completes."""
    from oracle import definition
    g = oir.generate(name, coll, n, **kw)
    pl = lower.lower(g, direct=True, pushreduce=True)
    count = 3000 + 7
    xs = inp.all_inputs("int32", 5, n, count * (n if coll == "reducescatter" else 1), mode="wrap")
    for inplace in (False, True):
        got = replay.replay(pl, xs, "int32", count, chunk_bytes=2048, instances=2, K=2, inplace=inplace)
        ref = {"allreduce": definition.allreduce, "allgather": lambda x, d: definition.allgather(x),
               "reducescatter": definition.reducescatter}[coll](xs, "int32")
        for r in range(n):
            assert np.array_equal(got[r], ref[r]), (inplace, r)
    for K, nmb in ((1, 2), (2, 3)):
        assert replay.happens_before_races(pl, n_mb=nmb, instances=1, K=K) == []
    assert replay.deadlock_free(pl, Ks=(1, 2), n_mbs=(1, 2, 3, 16))
