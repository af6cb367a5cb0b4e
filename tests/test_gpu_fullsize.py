"""Parity at BASELINE's full sizes in bench.py's launch configuration.

``test_fullsize_elementwise``: bench.py's N=1 workload (8 x 256 MiB bf16 ring AllReduce,
its exact launch geometry, out of place and in place) compared on EVERY element of every
rank's result with the oracle's step-order dataflow evaluation of the same IR
(``replay.dataflow_values``, pinned to the blocking replay in
``tests/test_oracle_pins_r2.py``), one algorithm chunk at a time on the host.

The other tests compare sampled outputs (random + chunk / micro-batch / instance-slice
boundaries) at sizes where a full host evaluation would take minutes."""
import numpy as np
import pytest

import resccl_inputs as inp
from oracle import ir as oir, replay

pytestmark = pytest.mark.gpu


def _positions(geo, c, rng, n_rand=3000):
    L = geo.chunk_len[c]
    if L == 0:
        return np.zeros(0, dtype=np.int64)
    pts = set(rng.integers(0, L, n_rand).tolist())
    for j in range(geo.n_mb):
        for i in range(geo.instances):
            lo, hi = geo.slice(c, j, i)
            for p in (lo, lo + 1, hi - 2, hi - 1):
                if 0 <= p < L:
                    pts.add(p)
    pts.update([0, L - 1])
    return np.array(sorted(pts), dtype=np.int64)


# bench.py's N=1 launch configuration (bench.py: instances 14 x 8 ranks = 112 CTAs)
BENCH_OPTS = dict(instances=14, chunkbytes=32 << 20, fifodepth=2, nwarps=8, direct=1, tmastages=2, tmatile=24576)


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


@pytest.mark.timeout(600)
@pytest.mark.parametrize("algo,n,size_mb,dtype,opts", [
    # the C2 sweep's largest size in the bench geometry
    ("ring", 8, 1024, "bfloat16", BENCH_OPTS),
    ("ring", 8, 256, "bfloat16", dict(instances=18, chunkbytes=4 << 20, fifodepth=2)),
    ("ring", 8, 256, "bfloat16", dict(instances=18, chunkbytes=4 << 20, fifodepth=2, direct=1)),
    ("ring", 8, 64, "float32", dict(instances=16, chunkbytes=2 << 20, fifodepth=2)),
    ("hm", 8, 64, "bfloat16", dict(instances=4, chunkbytes=1 << 20, fifodepth=2)),
    ("dbt", 8, 64, "float16", dict(instances=4, chunkbytes=1 << 20, fifodepth=2)),
])
def test_fullsize_sampled(algo, n, size_mb, dtype, opts):
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    elt = {"bfloat16": 2, "float16": 2, "float32": 4}[dtype]
    count = size_mb * (1 << 20) // elt
    opts = dict(opts)
    inplace = opts.pop("_inplace", False)
    g = oir.generate(algo, "allreduce", n, **({"g": 4} if algo == "hm" else {}))
    for k, v in opts.items():
        g.extra[k] = str(v)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(g.to_text())
        sends = [inp.rank_input_torch(dtype, 11, r, count) for r in range(n)]
        if inplace:  # one call: the result replaces the input
            grp.allreduce(sends, sends)
            torch.cuda.synchronize()
            recvs = sends
        else:
            recvs = [torch.empty_like(s) for s in sends]
            for _ in range(2):
                for t in recvs:
                    t.fill_(float("nan"))
                grp.allreduce(sends, recvs)
                torch.cuda.synchronize()
        assert grp.async_error() == 0
        geo = replay.Geometry("allreduce", n, count, elt, opts["chunkbytes"], opts["instances"])
        rng = np.random.default_rng(0)
        pos = [_positions(geo, c, rng) for c in range(n)]
        chunk_in = [[inp.rank_input_at(dtype, 11, r, c * geo.C + pos[c]) for c in range(n)] for r in range(n)]
        exp = replay.dataflow_values(g, chunk_in, dtype)
        for r in range(n):
            out = recvs[r]
            for c in range(n):
                if pos[c].size == 0:
                    continue
                idx = torch.from_numpy(c * geo.C + pos[c]).to(out.device)
                got = out[idx].cpu()
                got = got.view(torch.int16).numpy().view(np.uint16) if dtype == "bfloat16" else got.numpy()
                assert np.array_equal(got.view(np.uint8), exp[r][c].view(np.uint8)), (r, c)
    finally:
        grp.destroy()


@pytest.mark.timeout(600)
@pytest.mark.parametrize("name,coll,gkw,size_mb,dtype,opts", [
    ("ring", "allgather", {}, 1024, "bfloat16", dict(instances=18, chunkbytes=8 << 20, direct=1)),
    ("synth", "reducescatter", {"seed": 0, "fanout": 2}, 256, "float32", dict(instances=4, chunkbytes=1 << 20)),
    ("hm", "allreduce", {"g": 4}, 256, "bfloat16", dict(instances=4, chunkbytes=4 << 20, direct=1)),
])
def test_fullsize_sampled_ag_rs(name, coll, gkw, size_mb, dtype, opts):
    """Sampled parity at C2/C3/C4 sizes for AllGather (total output) and ReduceScatter
    (total input) and the hierarchical AllReduce in direct mode."""
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    elt = {"bfloat16": 2, "float16": 2, "float32": 4}[dtype]
    total = size_mb * (1 << 20) // elt
    cnt = total if coll == "allreduce" else total // n     # per-rank count argument
    send_n = cnt * n if coll == "reducescatter" else cnt
    recv_n = cnt * n if coll == "allgather" else cnt
    g = oir.generate(name, coll, n, **gkw)
    for k, v in opts.items():
        g.extra[k] = str(v)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(g.to_text())
        sends = [inp.rank_input_torch(dtype, 13, r, send_n) for r in range(n)]
        recvs = [torch.full((recv_n,), float("nan"), device="cuda:0", dtype=sends[0].dtype) for _ in range(n)]
        getattr(grp, coll)(sends, recvs)
        torch.cuda.synchronize()
        assert grp.async_error() == 0
        geo = replay.Geometry(coll, n, cnt, elt, opts["chunkbytes"], opts["instances"])
        rng = np.random.default_rng(1)
        pos = [_positions(geo, c, rng) for c in range(n)]
        chunk_in = []
        for r in range(n):
            row = []
            for c in range(n):
                if coll == "allgather":
                    row.append(inp.rank_input_at(dtype, 13, r, pos[c]) if r == c else None)
                else:
                    row.append(inp.rank_input_at(dtype, 13, r, geo.chunk_off("send", c) + pos[c]))
            chunk_in.append(row)
        exp = replay.dataflow_values(g, chunk_in, dtype)
        for r in range(n):
            for c in range(n):
                if coll == "reducescatter" and c != r:
                    continue
                idx = torch.from_numpy(geo.chunk_off("recv", c) + pos[c]).to(recvs[r].device)
                got = recvs[r][idx].cpu()
                got = got.view(torch.int16).numpy().view(np.uint16) if dtype == "bfloat16" else got.numpy()
                assert np.array_equal(got.view(np.uint8), exp[r][c].view(np.uint8)), (r, c)
    finally:
        grp.destroy()
