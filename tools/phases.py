"""Per-phase HBM efficiency on one B200 (8 virtual ranks, direct transport, bench
config): ring ReduceScatter (pull-reduce hops: 2 reads + 1 write per element), ring
AllGather (push hops: 1 read + 1 write) and AllReduce, against torch's own copy
(1R+1W) and add (2R+1W) kernels on 1 GiB operands as the attainable ceilings."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
OPTS = os.environ.get("PHASE_OPTS", "instances=36 nwarps=8 tmastages=3 tmatile=8192 chunkbytes=16777216 fifodepth=2 direct=1")


def timed(f, iters=10, warm=3):
    for _ in range(warm):
        f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters):
        f()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / iters * 1e-3


def coll_rate(coll, S):
    text = R.rescclGenerateIr("ring", coll, N, "")
    hdr, rest = text.split("\n", 1)
    grp = R.VirtualGroup(N, 0)
    grp.load(hdr + " " + OPTS + "\n" + rest)
    s_elems = S // 2
    if coll == "allreduce":
        sn = rn = s_elems
        per_hop = {"rs": 3, "ag": 2}
    elif coll == "allgather":
        sn, rn = s_elems // N, s_elems
    else:
        sn, rn = s_elems, s_elems // N
    s = [torch.randn(sn, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
    r = [torch.empty(rn, device="cuda:0", dtype=torch.bfloat16) for _ in range(N)]
    f = getattr(grp, coll)
    t = timed(lambda: f(s, r))
    chunk = S // N
    hops = N * (N - 1)
    traffic = {"allreduce": 5, "allgather": 2, "reducescatter": 3}[coll] * hops * chunk
    grp.destroy()
    return {"coll": coll, "S": S, "us": round(t * 1e6, 1), "hbm_gbs": round(traffic / t / 1e9, 1),
            "bus_gbs": round(S / t / 1e9 * (2 if coll == "allreduce" else 1) * (N - 1) / N, 1)}


out = []
for coll in ("reducescatter", "allgather", "allreduce"):
    out.append(coll_rate(coll, 256 << 20))
a = torch.randn(1 << 29, device="cuda:0").to(torch.bfloat16)
b = torch.randn(1 << 29, device="cuda:0").to(torch.bfloat16)
c = torch.empty_like(a)
t = timed(lambda: c.copy_(a))
out.append({"torch": "copy 1GiB bf16", "hbm_gbs": round(2 * a.numel() * 2 / t / 1e9, 1)})
t = timed(lambda: torch.add(a, b, out=c))
out.append({"torch": "add 1GiB bf16", "hbm_gbs": round(3 * a.numel() * 2 / t / 1e9, 1)})
for o in out:
    print(json.dumps(o), flush=True)
