"""Mid-size (4-32 MiB per rank) AllReduce schedule search on the device clock: the paper's
algorithms (ring, DBT, HM at g = 2 / 4 / 8) x link model x instances x transfer chunk; each
point is skipped when its CTAs do not fit co-resident.  One JSON line per point."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_sigcomm_liuhlgcwz025_b200 as R  # noqa: E402

N, REPS = 8, 20
SIZES = [4 << 20, 16 << 20, 32 << 20]


def graph_us(fn, st):
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
    pts = []
    for algo, gopt in (("hm", "g=2"), ("hm", "g=4"), ("hm", "g=8"), ("dbt", ""), ("ring", "")):
        for model in ("pair", "port"):
            for inst in (2, 4, 6, 9, 12, 16, 18):
                for cb in (1 << 20, 4 << 20):
                    pts.append((algo, gopt, f"instances={inst} nwarps=8 linkmodel={model} chunkbytes={cb} direct=1"))
    for algo, gopt, opts in pts:
        text = R.rescclGenerateIr(algo, "allreduce", N, gopt)
        h, rest = text.split("\n", 1)
        grp = R.VirtualGroup(N, 0)
        try:
            grp.load(h + " " + opts + "\n" + rest)
            for S in SIZES:
                cnt = S // 2
                s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
                r = [torch.empty_like(v) for v in s]
                grp.allreduce(s, r, stream=st)
                torch.cuda.synchronize()
                us = graph_us(lambda: grp.allreduce(s, r, stream=st), st)
                print(json.dumps({"algo": algo, "gopts": gopt, "opts": opts, "bytes": S, "graph_us": round(us, 2),
                                  "busbw_gbs": round(S / (us * 1e-6) / 1e9 * 2 * (N - 1) / N, 2),
                                  "err": grp.async_error()}), flush=True)
                del s, r
        except Exception as e:  # (too many CTAs for one launch, ...)
            print(json.dumps({"algo": algo, "gopts": gopt, "opts": opts, "skipped": str(e)[:120]}), flush=True)
        finally:
            grp.destroy()


if __name__ == "__main__":
    main()
