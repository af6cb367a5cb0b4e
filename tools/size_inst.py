"""Latency / busBW of ring AllReduce (8 virtual ranks, bf16, direct) vs message size for
several instance counts and transfer-chunk sizes: what a per-size algorithm choice could
gain.  python tools/size_inst.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
SIZES = [1 << k for k in range(10, 29, 2)]
CFGS = [dict(instances=i, chunkbytes=c) for i in (1, 2, 4, 8, 18) for c in (8 << 20,)]
CFGS += [dict(instances=18, chunkbytes=32 << 20), dict(instances=4, chunkbytes=32 << 20)]
text = R.rescclGenerateIr("ring", "allreduce", N)
h0, rest = text.split("\n", 1)
for cfg in CFGS:
    grp = R.VirtualGroup(N, 0)
    try:
        grp.load(h0 + "".join(f" {k}={v}" for k, v in cfg.items()) + " fifodepth=2 direct=1\n" + rest)
        for S in SIZES:
            cnt = S // 2
            s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
            r = [torch.empty_like(x) for x in s]
            for _ in range(3):
                grp.allreduce(s, r)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            it = 20 if S < (16 << 20) else 5
            e0.record()
            for _ in range(it):
                grp.allreduce(s, r)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / it
            print(json.dumps({**cfg, "bytes": S, "us": round(ms * 1e3, 1),
                              "busbw_gbs": round(S / (ms * 1e-3) / 1e9 * 2 * (N - 1) / N, 2),
                              "err": grp.async_error()}), flush=True)
            del s, r
    finally:
        grp.destroy()
