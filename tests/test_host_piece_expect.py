"""Pins the piecewise expectation the host-buffer GPU tests use (CPU only): for int32
every reduction order gives the same bits, so the concatenation of the oracle's
per-piece replays must equal the collective's plain definition for
AllReduce, AllGather (strided rows) and ReduceScatter (strided input rows)."""
import numpy as np
import pytest

from oracle import definition

import test_gpu_host_buffers as T


@pytest.mark.parametrize("coll", ["allreduce", "allgather", "reducescatter"])
@pytest.mark.parametrize("pe", [2048, 1000, 10 ** 6])
def test_piece_expectation_matches_definition(coll, pe):
    n, count = 4, 3 * 2048 + 513
    g, _ = T._text(coll, n, chunkbytes=2048, instances=2)
    xs = T._inputs(coll, "int32", n, count, 5)
    got = T._piece_expect(g, coll, xs, "int32", count, pe, n, chunk_bytes=2048, instances=2)
    ref = {"allreduce": lambda: definition.allreduce(xs, "int32"), "allgather": lambda: definition.allgather(xs),
           "reducescatter": lambda: definition.reducescatter(xs, "int32")}[coll]()
    for a, b in zip(got, ref):
        assert np.array_equal(a, b)
