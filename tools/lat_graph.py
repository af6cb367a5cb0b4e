"""Small-message AllReduce latency, eager vs CUDA-graph replay (device-side epochs):
ring, 8 virtual ranks, bf16.  python tools/lat_graph.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N, REPS = 8, 20
for inst in (1, 18):
    text = R.rescclGenerateIr("ring", "allreduce", N)
    h, rest = text.split("\n", 1)
    grp = R.VirtualGroup(N, 0)
    grp.load(h + f" instances={inst} chunkbytes={8 << 20} direct=1\n" + rest)
    for S in (1024, 65536, 1 << 20, 16 << 20):
        cnt = S // 2
        s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
        r = [torch.empty_like(x) for x in s]
        st = torch.cuda.Stream()
        with torch.cuda.stream(st):
            for _ in range(3):
                grp.allreduce(s, r, stream=st)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(REPS):
            grp.allreduce(s, r, stream=st)
        e1.record(st)
        torch.cuda.synchronize()
        eager = e0.elapsed_time(e1) / REPS
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(REPS):
                grp.allreduce(s, r, stream=st)
        g.replay()
        torch.cuda.synchronize()
        e0.record(st)
        with torch.cuda.stream(st):
            g.replay()
        e1.record(st)
        torch.cuda.synchronize()
        graph = e0.elapsed_time(e1) / REPS
        print(json.dumps({"instances": inst, "bytes": S, "eager_us": round(eager * 1e3, 1),
                          "graph_us": round(graph * 1e3, 1), "err": grp.async_error()}), flush=True)
    grp.destroy()
