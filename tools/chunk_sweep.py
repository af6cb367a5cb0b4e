"""busBW vs transfer-chunk size (micro-batch bytes) for ring AllReduce on 8 virtual ranks:
mid-size messages are bounded by the per-hop fill/drain when a hop is one micro-batch.
  python tools/chunk_sweep.py  (env CS_SIZES MiB list, CS_CHUNKS KiB list, CS_INST)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
SIZES = [float(x) for x in os.environ.get("CS_SIZES", "4,16,64,256").split(",")]
CHUNKS = [int(x) for x in os.environ.get("CS_CHUNKS", "256,512,1024,2048,4096,8192,32768").split(",")]
INST = int(os.environ.get("CS_INST", "18"))
EXTRA = os.environ.get("CS_OPTS", "")
for mib in SIZES:
    S = int(mib * (1 << 20))
    cnt = S // 2
    s = [(torch.rand(cnt, device="cuda:0") * 2 - 1).to(torch.bfloat16) for _ in range(N)]
    r = [torch.empty_like(x) for x in s]
    for ck in CHUNKS:
        text = R.rescclGenerateIr("ring", "allreduce", N)
        h, rest = text.split("\n", 1)
        h += f" instances={INST} chunkbytes={ck << 10} fifodepth=2 direct=1 " + EXTRA
        grp = R.VirtualGroup(N, 0)
        try:
            grp.load(h + "\n" + rest)
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
            bus = S / (ms * 1e-3) / 1e9 * 2 * (N - 1) / N
            print(json.dumps({"MiB": mib, "chunk_kib": ck, "instances": INST, "us": round(ms * 1e3, 1),
                              "busbw_gbs": round(bus, 1), "opts": EXTRA, "err": grp.async_error()}), flush=True)
        finally:
            grp.destroy()
