"""Parity at BASELINE's full sizes in bench.py's launch configuration.

``test_fullsize_elementwise``: bench.py's N=1 workload (8 x 256 MiB bf16 ring AllReduce,
its exact launch geometry, out of place and in place) compared on EVERY element of every
rank's result with the oracle's step-order dataflow evaluation of the same IR
(``replay.dataflow_values``, pinned to the blocking replay in
``tests/test_oracle_pins_r2.py``), one algorithm chunk at a time on the host.

``test_fullsize_fast``: every other full-size configuration (C2's 1 GiB, C3's DBT / HM,
C4's synthesized AllGather / ReduceScatter, the staged transport) compared on EVERY
element with the C++ fast replay (``oracle/fastreplay.cc``, pinned to the Python replay
in ``tests/test_oracle_fast.py``).  Its inputs are the shared recipe evaluated by torch
(``resccl_inputs.rank_input_torch``, pinned bit-identical to the numpy recipe in
``tests/test_inputs.py``) and copied to the host before the collective runs."""
import os

import numpy as np
import pytest

import resccl_inputs as inp
from oracle import fastreplay, ir as oir, replay

pytestmark = pytest.mark.gpu


# bench.py's N=1 launch configuration (bench.py: instances 12 x 8 ranks = 96 CTAs of 384 threads)
BENCH_OPTS = dict(instances=12, chunkbytes=32 << 20, fifodepth=2, nwarps=12, direct=1, tmastages=2, tmatile=28672)


@pytest.mark.timeout(900)
@pytest.mark.parametrize("inplace", [False, True])
def test_fullsize_elementwise(inplace):
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n, dtype, seed = 8, "bfloat16", 11
    count = 256 * (1 << 20) // 2
    g = oir.generate("ring", "allreduce", n)
    for k, v in BENCH_OPTS.items():
        g.extra[k] = str(v)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(g.to_text())
        sends = [inp.rank_input_torch(dtype, seed, r, count) for r in range(n)]
        recvs = sends if inplace else [torch.full_like(s, float("nan")) for s in sends]
        grp.allreduce(sends, recvs)
        torch.cuda.synchronize()
        assert grp.async_error() == 0
        geo = replay.Geometry("allreduce", n, count, 2, BENCH_OPTS["chunkbytes"], BENCH_OPTS["instances"])
        checked = 0
        for c in range(n):
            L = geo.chunk_len[c]
            if L == 0:
                continue
            # chunk c of every rank's input, straight from the shared recipe (numpy)
            ci = [[inp.rank_input(dtype, seed, r, L, offset=c * geo.C) if cc == c else np.zeros(0, np.uint16)
                   for cc in range(n)] for r in range(n)]
            exp = replay.dataflow_values(g, ci, dtype)
            for r in range(n):
                got = recvs[r][c * geo.C:c * geo.C + L].cpu().view(torch.int16).numpy().view(np.uint16)
                bad = np.flatnonzero(got != exp[r][c])
                assert bad.size == 0, (r, c, bad[:5], got[bad[:5]], exp[r][c][bad[:5]])
                checked += L
        assert checked == n * count  # every element of every rank
    finally:
        grp.destroy()


@pytest.mark.timeout(900)
@pytest.mark.parametrize("name,coll,gkw,size_mb,dtype,opts", [
    # the C2 sweep's largest size in the bench geometry, AllReduce and AllGather (total output)
    ("ring", "allreduce", {}, 1024, "bfloat16", BENCH_OPTS),
    ("ring", "allgather", {}, 1024, "bfloat16", dict(instances=18, chunkbytes=8 << 20, direct=1)),
    # staged FIFO transport and the library-default geometry
    ("ring", "allreduce", {}, 256, "bfloat16", dict(instances=18, chunkbytes=4 << 20, fifodepth=2)),
    ("ring", "allreduce", {}, 64, "float32", dict(instances=16, chunkbytes=2 << 20, fifodepth=2)),
    # C3: hierarchical 2x4 and double binary tree
    ("hm", "allreduce", {"g": 4}, 256, "bfloat16", dict(instances=4, chunkbytes=4 << 20, direct=1)),
    ("hm", "allreduce", {"g": 4}, 64, "bfloat16", dict(instances=4, chunkbytes=1 << 20, fifodepth=2)),
    ("dbt", "allreduce", {}, 256, "bfloat16", dict(instances=2, chunkbytes=4 << 20, direct=1)),
    ("dbt", "allreduce", {}, 64, "float16", dict(instances=4, chunkbytes=1 << 20, fifodepth=2)),
    # the size-tuned classes bench.py selects: 2x4 hierarchical at 4 MiB, the
    # full mesh under the port model at 16 MiB (18 instances) and 256 MiB (16 instances)
    ("hm", "allreduce", {"g": 4}, 4, "bfloat16", dict(instances=4, chunkbytes=512 << 10, nwarps=8, direct=1)),
    ("hm", "allreduce", {"g": 8}, 16, "bfloat16", dict(instances=18, chunkbytes=8 << 20, nwarps=8,
                                                       linkmodel="port", direct=1)),
    ("hm", "allreduce", {"g": 8}, 256, "bfloat16", dict(instances=16, chunkbytes=8 << 20, nwarps=8,
                                                        linkmodel="port", direct=1)),
    # C4: synthesized AllGather / ReduceScatter (total buffer sizes)
    ("synth", "reducescatter", {"seed": 0, "fanout": 2}, 256, "float32", dict(instances=4, chunkbytes=1 << 20)),
    ("synth", "allgather", {"seed": 1, "fanout": 3}, 256, "bfloat16", dict(instances=3, chunkbytes=4 << 20, direct=1)),
])
def test_fullsize_fast(name, coll, gkw, size_mb, dtype, opts):
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    elt = {"bfloat16": 2, "float16": 2, "float32": 4}[dtype]
    total = size_mb * (1 << 20) // elt
    cnt = total if coll == "allreduce" else total // n     # the collective's count argument
    send_n = cnt * n if coll == "reducescatter" else cnt
    recv_n = cnt * n if coll == "allgather" else cnt
    g = oir.generate(name, coll, n, **gkw)
    for k, v in opts.items():
        g.extra[k] = str(v)
    sends = [inp.rank_input_torch(dtype, 13, r, send_n) for r in range(n)]
    host_in = [(s.cpu().view(torch.int16).numpy().view(np.uint16) if dtype == "bfloat16" else s.cpu().numpy())
               for s in sends]
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(g.to_text())
        recvs = [torch.full((recv_n,), float("nan"), device="cuda:0", dtype=sends[0].dtype) for _ in range(n)]
        getattr(grp, coll)(sends, recvs)
        torch.cuda.synchronize()
        assert grp.async_error() == 0
        got = [(t.cpu().view(torch.int16).numpy().view(np.uint16) if dtype == "bfloat16" else t.cpu().numpy())
               for t in recvs]
    finally:
        grp.destroy()
    del sends, recvs
    exp = fastreplay.replay_full(g, host_in, dtype, cnt, threads=max(1, min(32, os.cpu_count() or 1)))
    for r in range(n):
        bad = np.flatnonzero(got[r].view(np.uint8) != exp[r].view(np.uint8))
        assert bad.size == 0, (r, bad.size, bad[:5])
