"""AllReduce latency / busBW vs size on the device clock: 20 calls captured in one CUDA
graph (device-side epochs) and replayed, so host submission cost is excluded (an eager
loop of 8 virtual ranks is host-bound below ~1 MiB: ~60 us of ctypes + runtime calls per
group call).  Ring (or PHASE_ALGO), 8 virtual ranks, bf16.

    python tools/lat_graph.py "opts A" "opts B" ...      (env LAT_SIZES="[1024, ...]")
Prints one JSON line per (opts, size); also a reference line for 20 empty torch kernels."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_sigcomm_liuhlgcwz025_b200 as R  # noqa: E402

N, REPS = int(os.environ.get("LAT_N", "8")), 20
ALGO = os.environ.get("LAT_ALGO", "ring")
GOPTS = os.environ.get("LAT_GOPTS", "g=4" if ALGO == "hm" else "")
OPTS = sys.argv[1:] or ["instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1"]
SIZES = [int(x) for x in os.environ.get("LAT_SIZES", "[1024, 65536, 1048576, 16777216, 67108864]")[1:-1].split(",")]


def graph_time(fn, st):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        for _ in range(REPS):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best = None
    for _ in range(3):
        e0.record(st)
        with torch.cuda.stream(st):
            g.replay()
        e1.record(st)
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / REPS * 1e3
        best = t if best is None else min(best, t)
    return best


def main():
    st = torch.cuda.Stream()
    x = torch.zeros(1, device="cuda:0")
    print(json.dumps({"reference": "empty torch kernel in a graph", "us": round(graph_time(lambda: x.add_(1), st), 2)}),
          flush=True)
    for opts in OPTS:
        text = R.rescclGenerateIr(ALGO, "allreduce", N, GOPTS)
        h, rest = text.split("\n", 1)
        grp = R.VirtualGroup(N, 0)
        grp.load(h + " " + opts + "\n" + rest)
        for S in SIZES:
            cnt = S // 2
            s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
            r = [torch.empty_like(v) for v in s]
            for _ in range(3):
                grp.allreduce(s, r, stream=st)
            torch.cuda.synchronize()
            us = graph_time(lambda: grp.allreduce(s, r, stream=st), st)
            bus = S / (us * 1e-6) / 1e9 * 2 * (N - 1) / N
            print(json.dumps({"opts": opts, "algo": ALGO, "gopts": GOPTS, "bytes": S, "graph_us": round(us, 2),
                              "busbw_gbs": round(bus, 2), "err": grp.async_error()}), flush=True)
            del s, r
        grp.destroy()


if __name__ == "__main__":
    main()
