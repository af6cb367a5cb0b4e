"""Pins of the C++ fast replay (oracle/fastreplay.cc).

* equal, byte for byte, to the Python blocking replay of the lowered plan
  (``replay.replay``) for every algorithm of the pin suite, four dtypes, ragged counts,
  1 and several threads;
* int32 (any schedule) equal to the definition, with wraparound;
* its own fp16 rounding equal to numpy's on every finite half bit pattern pair sum
  sampled (the step that could silently differ from the Python replay's arithmetic).
"""
import numpy as np
import pytest

import resccl_inputs as inp
from oracle import definition, fastreplay, ir as oir, lower, replay

ALGOS = [
    ("ring", "allreduce", 2, {}), ("ring", "allreduce", 8, {}), ("ring", "allgather", 5, {}),
    ("ring", "reducescatter", 4, {}), ("dbt", "allreduce", 8, {}), ("dbt", "allreduce", 5, {}),
    ("hm", "allreduce", 8, {"g": 4}), ("hm", "allgather", 8, {"g": 4}),
    ("synth", "allgather", 6, {"seed": 1, "fanout": 2}), ("synth", "reducescatter", 8, {"seed": 0, "fanout": 2}),
]


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
@pytest.mark.parametrize("dtype", ["int32", "float32", "float16", "bfloat16"])
def test_fast_replay_equals_python_replay(name, coll, n, kw, dtype):
    g = oir.generate(name, coll, n, **kw)
    pl = lower.lower(g)
    for count, threads in ((1, 1), (4097, 3), (70000 + 5, 4)):
        xs = inp.all_inputs(dtype, 9, n, count * (n if coll == "reducescatter" else 1))
        exp = replay.replay(pl, xs, dtype, count, chunk_bytes=1 << 16, instances=2, K=2)
        got = fastreplay.replay_full(g, xs, dtype, count, threads=threads)
        for r in range(n):
            a = got[r].view(np.uint8)
            b = np.ascontiguousarray(exp[r]).view(np.uint8)
            assert np.array_equal(a, b), (count, r)


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
def test_fast_replay_int32_wrap_equals_definition(name, coll, n, kw):
    g = oir.generate(name, coll, n, **kw)
    count = 10007
    xs = inp.all_inputs("int32", 4, n, count * (n if coll == "reducescatter" else 1), mode="wrap")
    got = fastreplay.replay_full(g, xs, "int32", count, threads=2)
    ref = {"allreduce": definition.allreduce, "allgather": lambda x, d: definition.allgather(x),
           "reducescatter": definition.reducescatter}[coll](xs, "int32")
    for r in range(n):
        assert np.array_equal(got[r], ref[r])


def test_fast_replay_in_place_allreduce():
    g = oir.generate("ring", "allreduce", 4)
    xs = inp.all_inputs("bfloat16", 2, 4, 5000)
    exp = fastreplay.replay_full(g, [x.copy() for x in xs], "bfloat16", 5000)
    bufs = [x.copy() for x in xs]
    fastreplay.replay_full(g, bufs, "bfloat16", 5000, outputs=bufs)
    for r in range(4):
        assert np.array_equal(bufs[r], exp[r])


def test_fast_replay_f16_rounding_matches_numpy_on_sampled_pairs():
    """fp16 sums through the replay's own float->half conversion == numpy's RNE, on
    2^20 random bit-pattern pairs (normals, subnormals, overflow to inf, ties)."""
    rng = np.random.default_rng(0)
    a = rng.integers(0, 1 << 16, 1 << 20, dtype=np.uint16)
    b = rng.integers(0, 1 << 16, 1 << 20, dtype=np.uint16)
    fin = (np.abs(a.view(np.float16)) < np.inf) & (np.abs(b.view(np.float16)) < np.inf)
    a, b = a[fin], b[fin]
    with np.errstate(over="ignore"):
        want = (a.view(np.float16).astype(np.float32) + b.view(np.float16).astype(np.float32)).astype(np.float16)
    g = oir.IR("pair", "allreduce", 2, 2, [oir.Transfer(1, 0, 0, 0, "rrc")])
    # chunk 0 of rank 0 := rank0 (+) rank1 on the first C elements: use count = 2C so
    # chunk 0 covers exactly the first half
    n = a.size
    C = -(-n // 128) * 128
    x0 = np.zeros(2 * C, np.float16)
    x1 = np.zeros(2 * C, np.float16)
    x0[:n] = a.view(np.float16)
    x1[:n] = b.view(np.float16)
    out = fastreplay.replay_full(g, [x0, x1], "float16", 2 * C)
    got = out[0][:n]
    assert np.array_equal(got.view(np.uint16), want.view(np.uint16))
