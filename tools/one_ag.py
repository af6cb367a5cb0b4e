"""One ring AllGather (8 virtual ranks, bf16, 256 MiB total, direct) at a given instance
count -- the target of an ncu source-level capture of the lane engine's copy path.
  python tools/one_ag.py [instances] [coll] [extra opts]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
inst = int(sys.argv[1]) if len(sys.argv) > 1 else 1
coll = sys.argv[2] if len(sys.argv) > 2 else "allgather"
extra = " ".join(sys.argv[3:])
S = 256 << 20
cnt = S // 2
sn, rn = {"allreduce": (cnt, cnt), "allgather": (cnt // N, cnt), "reducescatter": (cnt, cnt // N)}[coll]
s = [torch.randn(sn, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
r = [torch.empty(rn, device="cuda:0", dtype=torch.bfloat16) for _ in range(N)]
text = R.rescclGenerateIr("ring", coll, N)
h, rest = text.split("\n", 1)
h += f" instances={inst} chunkbytes={32 << 20} fifodepth=2 direct=1 nwarps=16 tmastages=2 tmatile=24576 {extra}"
grp = R.VirtualGroup(N, 0)
grp.load(h + "\n" + rest)
for _ in range(3):
    getattr(grp, coll)(s, r)
torch.cuda.synchronize()
print("err", grp.async_error())
grp.destroy()
