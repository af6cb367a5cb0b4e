"""Ad-hoc engine throughput probe: one collective on N virtual ranks, in-place or not.
usage: python tools/exp_ag.py coll N S_MiB inplace(0/1) "opts" [trace]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

coll, N, S, inplace, opts = sys.argv[1], int(sys.argv[2]), int(float(sys.argv[3]) * (1 << 20)), int(sys.argv[4]), sys.argv[5]
trace = len(sys.argv) > 6
text = R.rescclGenerateIr("ring", coll, N)
h, rest = text.split("\n", 1)
grp = R.VirtualGroup(N, 0)
grp.load(h + " " + opts + (" trace=1" if trace else "") + "\n" + rest)
info = grp.plan_info()
e = S // 2
if coll == "allgather":
    big = [torch.randn(e, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
    seg = e // N
    s = [big[r][r * seg:(r + 1) * seg] if inplace else torch.randn(seg, device="cuda:0").to(torch.bfloat16) for r in range(N)]
    rr = big
elif coll == "reducescatter":
    s = [torch.randn(e, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
    seg = e // N
    rr = [s[r][r * seg:(r + 1) * seg] if inplace else torch.empty(seg, device="cuda:0", dtype=torch.bfloat16) for r in range(N)]
else:
    s = [torch.randn(e, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
    rr = s if inplace else [torch.empty_like(x) for x in s]
f = getattr(grp, coll)
for _ in range(3):
    f(s, rr)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    f(s, rr)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 5
hb = {"allreduce": 5.0, "reducescatter": 3.0, "allgather": 2.0}[coll] * (N - 1) / N * S * N
blocks = sum(info["blocks_per_rank"])
out = {"coll": coll, "N": N, "S": S, "inplace": inplace, "opts": opts, "us": round(ms * 1e3, 1), "blocks": blocks,
       "hbm_gbs": round(hb / ms / 1e6, 1), "per_cta_gbs": round(hb / ms / 1e6 / blocks, 1), "err": grp.async_error()}
if trace:
    u = R.rescclGetTbUtilization(grp.comms[0].algos[-1])
    out.update({k: u[k] for k in ("comm_time", "avg_idle", "max_idle", "span_ns") if k in u})
print(json.dumps(out), flush=True)
grp.destroy()
