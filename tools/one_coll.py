"""Run one collective on 8 virtual ranks a few times (ncu target).
usage: python tools/one_coll.py coll size_mb "opts" iters [algo] [generator opts]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R
coll, S, opts, iters = sys.argv[1], int(float(sys.argv[2]) * (1 << 20)), sys.argv[3], int(sys.argv[4])
N = 8
algo = sys.argv[5] if len(sys.argv) > 5 else "ring"
gopts = sys.argv[6] if len(sys.argv) > 6 else ""
text = R.rescclGenerateIr(algo, coll, N, gopts)
hdr, rest = text.split("\n", 1)
grp = R.VirtualGroup(N, 0)
grp.load(hdr + " " + opts + "\n" + rest)
e = S // 2
sn, rn = {"allreduce": (e, e), "allgather": (e // N, e), "reducescatter": (e, e // N)}[coll]
s = [torch.randn(sn, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
r = [torch.empty(rn, device="cuda:0", dtype=torch.bfloat16) for _ in range(N)]
for _ in range(iters):
    getattr(grp, coll)(s, r)
torch.cuda.synchronize()
print("err", grp.async_error())
