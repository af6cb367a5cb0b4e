"""Measurement sweeps on one B200 (8 virtual ranks), one JSON line per point:
  c2     ring allreduce / allgather, 1 KiB .. 1 GiB, bf16 / fp32 / int32   (BASELINE configs[1])
  c3     DBT and HM 2x4 allreduce under a TB budget 1..16                   (configs[2])
  c4     synthesized allgather / reducescatter, 4..256 MiB, fanout 2/3      (configs[3])
  f2     HPDS vs round-robin sub-pipelines (Fig. 10b analogue)
  nr     ring allreduce bf16 at 2 / 4 / 8 virtual ranks vs size (the metric's 2/4/8 axis), the
         bench geometry with 148 // N instances per rank (every SM busy at every N)
  geo    DBT / HM 2x4 allreduce and synthesized AG / RS at 256 MiB under transfer-chunk,
         instance and warp-count variants (the non-ring schedules' geometry search)
busBW follows nccl-tests: AR 2(N-1)/N, AG/RS (N-1)/N of algBW, S = per-rank buffer
(AG: total output; RS: total input).  Usage: python tools/sweep.py c2 [c3 c4 f2]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
GRAPH = os.environ.get("SWEEP_GRAPH", "1") == "1"  # device-clock timing (CUDA-graph replay)
BASE = dict(instances=14, chunkbytes=32 << 20, fifodepth=2, nwarps=8, direct=int(os.environ.get("SWEEP_DIRECT", "1")))
ELT = {"bfloat16": 2, "float32": 4, "int32": 4}


def measure(name, coll, gopts, opts, S, dtype="bfloat16", iters=10, warm=3, n=None):
    global N
    N0, N = N, (n or N)
    try:
        return _measure(name, coll, gopts, opts, S, dtype, iters, warm)
    finally:
        N = N0


def _measure(name, coll, gopts, opts, S, dtype="bfloat16", iters=10, warm=3):
    text = R.rescclGenerateIr(name, coll, N, gopts)
    hdr, rest = text.split("\n", 1)
    hdr += "".join(f" {k}={v}" for k, v in opts.items())
    grp = R.VirtualGroup(N, 0)
    try:
        grp.load(hdr + "\n" + rest)
        info = grp.plan_info()
        elt = ELT[dtype]
        if coll == "allreduce":
            cnt = S // elt
            sn, rn = cnt, cnt
        elif coll == "allgather":
            cnt = S // elt // N
            sn, rn = cnt, cnt * N
        else:
            cnt = S // elt // N
            sn, rn = cnt * N, cnt
        tdt = getattr(torch, dtype)
        if tdt.is_floating_point:
            s = [torch.randn(sn, device="cuda:0").to(tdt) for _ in range(N)]
        else:
            s = [torch.randint(-1000, 1000, (sn,), device="cuda:0", dtype=tdt) for _ in range(N)]
        r = [torch.empty(rn, device="cuda:0", dtype=tdt) for _ in range(N)]
        f = getattr(grp, coll)
        for _ in range(warm):
            f(s, r)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if GRAPH:
            # device clock: the calls captured in one CUDA graph and replayed (an eager loop
            # of 8 virtual-rank calls is host-bound below ~1 MiB)
            st = torch.cuda.Stream()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=st):
                for _ in range(iters):
                    f(s, r, stream=st) if coll == "allgather" else f(s, r, "sum", stream=st)
            g.replay()
            torch.cuda.synchronize()
            e0.record(st)
            with torch.cuda.stream(st):
                g.replay()
            e1.record(st)
            torch.cuda.synchronize()
            del g
        else:
            e0.record()
            for _ in range(iters):
                f(s, r)
            e1.record()
            torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / iters
        err = grp.async_error()
        Sb = (sn if coll != "allgather" else rn) * elt
        alg = Sb / (ms * 1e-3) / 1e9
        bus = alg * (2 * (N - 1) / N if coll == "allreduce" else (N - 1) / N)
        return {"nranks": N, "algo": name, "coll": coll, "gopts": gopts, "opts": opts, "dtype": dtype, "bytes": Sb,
                "us": round(ms * 1e3, 2), "algbw_gbs": round(alg, 2), "busbw_gbs": round(bus, 2),
                "ctas_per_rank": info["ctas"], "blocks": sum(info["blocks_per_rank"]),
                "instances": info["instances"], "linkmodel": info["linkmodel"], "fused": info["plan"]["fused"],
                "sched": info.get("sched"), "direct": info.get("direct"), "err": err,
                "timing": "graph" if GRAPH else "eager"}
    finally:
        grp.destroy()


def emit(d):
    print(json.dumps(d), flush=True)


which = sys.argv[1:] or ["c2"]
if "c2" in which:
    for coll in ("allreduce", "allgather"):
        for dtype in ("bfloat16", "float32", "int32"):
            sizes = [1 << k for k in range(10, 31, 2)] if dtype == "bfloat16" else [1 << 20, 64 << 20, 256 << 20]
            for S in sizes:
                emit(measure("ring", coll, "", BASE, S, dtype, iters=20 if S < (16 << 20) else 10))
if "c3" in which:
    # TB budget B = CTAs per rank (instances = floor(B / T_min) under the pair model, the
    # port model below T_min); each schedule's best transfer chunk of the r02 geometry
    # sweep (DBT 8 MiB, HM 1 MiB), 256-thread CTAs
    for name, g, cb, lm in (("dbt", "", 8 << 20, None), ("hm", "g=4", 1 << 20, None), ("dbt", "", 8 << 20, "port"),
                            ("hm", "g=4", 1 << 20, "port")):
        for budget in (1, 2, 4, 8, 12, 16, 18):
            for S in (64 << 20, 256 << 20):
                o = dict(chunkbytes=cb, fifodepth=2, tbbudget=budget, nwarps=8, direct=BASE["direct"])
                if lm:
                    o["linkmodel"] = lm
                emit(measure(name, "allreduce", g, o, S))
    for S in (64 << 20, 256 << 20):
        emit(measure("ring", "allreduce", "", dict(chunkbytes=1 << 20, fifodepth=2, instances=2,
                                                   direct=BASE["direct"]), S))
if "c3w" in which:
    # the C3 budget sweep at the r02 per-SM geometry (12 warps, 28 KiB tiles), DBT under the
    # port link model and HM 2x4 under the pair model (each one's better model, §5.13)
    for name, g, cb, lm in (("dbt", "", 8 << 20, "port"), ("hm", "g=4", 1 << 20, None)):
        for budget in (4, 8, 12, 16, 18):
            o = dict(chunkbytes=cb, fifodepth=2, tbbudget=budget, nwarps=12, tmatile=28672, direct=BASE["direct"])
            if lm:
                o["linkmodel"] = lm
            emit(measure(name, "allreduce", g, o, 256 << 20))
if "c4w" in which:
    # synthesized AG / RS at 256 MiB: instances x transfer chunk at 12 warps, 28 KiB tiles
    for coll in ("allgather", "reducescatter"):
        for inst in (3, 4):
            for cb in (2 << 20, 8 << 20):
                emit(measure("synth", coll, "seed=0 fanout=2", dict(instances=inst, chunkbytes=cb, fifodepth=2,
                                                                     nwarps=12, tmatile=28672,
                                                                     direct=BASE["direct"]), 256 << 20))
if "c4" in which:
    for coll in ("allgather", "reducescatter"):
        for fan in (2, 3):
            for S in (4 << 20, 16 << 20, 64 << 20, 256 << 20):
                emit(measure("synth", coll, f"seed=0 fanout={fan}", dict(instances=4, chunkbytes=1 << 20,
                                                                          fifodepth=2, direct=BASE["direct"]), S))
if "f2" in which:
    for name, coll, g in (("hm", "allreduce", "g=4"), ("hm", "allgather", "g=4"), ("dbt", "allreduce", ""),
                          ("synth", "allgather", "seed=0 fanout=2"), ("synth", "reducescatter", "seed=1 fanout=3")):
        for sched in ("hpds", "rr"):
            emit(measure(name, coll, g, dict(instances=4, chunkbytes=1 << 20, fifodepth=2, sched=sched,
                                             direct=BASE["direct"]), 64 << 20))
if "nr" in which:
    for n in (2, 4, 8):
        for S in [1 << k for k in range(20, 31, 2)]:
            emit(measure("ring", "allreduce", "", dict(instances=min(64, 148 // n), chunkbytes=32 << 20, fifodepth=2,
                                                       nwarps=8, direct=BASE["direct"]), S,
                         iters=20 if S < (64 << 20) else 10, n=n))
if "geo" in which:
    # instance counts keep every launch co-resident (<= 148 CTAs of one SM each)
    for name, coll, g, insts in (("dbt", "allreduce", "", (4, 6)), ("hm", "allreduce", "g=4", (2, 4)),
                                 ("synth", "allgather", "seed=0 fanout=2", (2, 4)),
                                 ("synth", "reducescatter", "seed=0 fanout=2", (2, 4))):
        for cb in (1 << 20, 4 << 20, 8 << 20, 32 << 20):
            for inst in insts:
                for nw in (8, 16):
                    emit(measure(name, coll, g, dict(instances=inst, chunkbytes=cb, fifodepth=2, nwarps=nw,
                                                     direct=BASE["direct"]), 256 << 20))
