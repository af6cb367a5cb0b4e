"""SMs used vs bandwidth (the Fig. 4 analogue on one B200): ring AllReduce,
8 virtual ranks, bf16, S MiB per rank, direct transport, for a range of instance counts
(CTAs per rank).  One JSON line per point: busBW, HBM rate (5(N-1)/N * S * N algorithmic
bytes) and the SMs the launch occupies.

  python tools/sm_budget.py [S_MiB] [geometry ...]
geometry: "two" = 256-thread CTAs, 2 x 12 KiB-tile stages (two CTAs per SM);
          "one" = 512-thread CTAs, 4 x 16 KiB-tile stages (one CTA per SM)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
S = int(float(sys.argv[1]) * (1 << 20)) if len(sys.argv) > 1 else 256 << 20
GEOS = sys.argv[2:] or ["two", "one"]
GEO = {"two": dict(nwarps=8, tmastages=2, tmatile=12288), "one": dict(nwarps=16, tmastages=4, tmatile=16384)}
EXTRA = os.environ.get("SMB_OPTS", "")
INST = [int(x) for x in os.environ.get("SMB_INST", "1,2,3,4,6,8,10,12,16,18,24,30,37").split(",")]
n_sm = torch.cuda.get_device_properties(0).multi_processor_count

cnt = S // 2
s = [(torch.rand(cnt, device="cuda:0") * 2 - 1).to(torch.bfloat16) for _ in range(N)]
r = [torch.empty_like(x) for x in s]
for geo in GEOS:
    for inst in INST:
        if geo == "one" and inst * N > n_sm:
            continue
        if inst * N > 2 * n_sm:
            continue
        cb = max(1 << 20, min(32 << 20, S // N))
        opts = dict(instances=inst, chunkbytes=cb, fifodepth=2, direct=1, **GEO[geo])
        text = R.rescclGenerateIr("ring", "allreduce", N)
        h, rest = text.split("\n", 1)
        h += "".join(f" {k}={v}" for k, v in opts.items()) + (" " + EXTRA if EXTRA else "")
        grp = R.VirtualGroup(N, 0)
        try:
            grp.load(h + "\n" + rest)
            info = grp.plan_info()
            for _ in range(3):
                grp.allreduce(s, r)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            it = 10
            e0.record()
            for _ in range(it):
                grp.allreduce(s, r)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / it
            blocks = sum(info["blocks_per_rank"])
            bus = S / (ms * 1e-3) / 1e9 * 2 * (N - 1) / N
            hbm = 5.0 * (N - 1) / N * S * N / (ms * 1e-3) / 1e9
            print(json.dumps({"geometry": geo, "instances": inst, "ctas": blocks,
                              "sms": min(n_sm, blocks),
                              "S": S, "us": round(ms * 1e3, 1), "busbw_gbs": round(bus, 1),
                              "hbm_gbs": round(hbm, 1), "per_sm_hbm_gbs": round(hbm / min(n_sm, blocks), 1),
                              "opts": EXTRA, "err": grp.async_error()}), flush=True)
        finally:
            grp.destroy()
