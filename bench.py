#!/usr/bin/env python
"""ResCCL bench: AllReduce bus bandwidth of the generated primitive-level kernels.

Contract (see the task's bench.py section):
  python bench.py --gpus N --steps K --warmup W [--impl resccl|reference]
prints ONE JSON line on rank 0.

Workload
  N = 1  (default): BASELINE configs[1]'s ring AllReduce at 8 ranks, run as 8 virtual
         ranks on cuda:0 (every rank's buffers and FIFOs in one B200's HBM; one
         generated kernel holds all ranks' CTAs).  bf16, 256 MiB per rank.
  N > 1  (torchrun, one process per GPU): N real ranks over CUDA-IPC peer memory
         (NVLink), same algorithm and per-rank size.
A step = one AllReduce of the whole buffer (every §8(a) row of the hot path runs in
it: IR -> plan are load-time; the generated kernel's primitives are the step).

busBW = algBW * 2(N-1)/N with algBW = S / t (nccl-tests convention).
Inputs are larger than L2 (126 MB) on every rank, so no L2 flush is needed.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="resccl", choices=["resccl", "reference"])
    p.add_argument("--algo", default="ring", choices=["ring", "dbt", "hm"])
    p.add_argument("--vranks", type=int, default=8, help="virtual ranks at --gpus 1")
    p.add_argument("--size-mb", type=float, default=256.0, help="MiB per rank")
    p.add_argument("--dtype", default="bfloat16", choices=["bfloat16", "float32", "float16", "int32"])
    p.add_argument("--instances", type=int, default=0, help="0 = auto")
    p.add_argument("--chunk-bytes", type=int, default=0)
    p.add_argument("--fifo-depth", type=int, default=0)
    p.add_argument("--nwarps", type=int, default=0)
    p.add_argument("--tma", type=int, default=-1, help="-1 = library default (on)")
    p.add_argument("--direct", type=int, default=-1, help="direct push/pull transport (default 1; N>1 registers a symmetric window)")
    p.add_argument("--nccl-compare", type=int, default=1,
                   help="N>1: also report a traced call's TB utilisation and NCCL's same-size AllReduce (busBW, "
                        "channels)")
    p.add_argument("--pushreduce", type=int, default=0,
                   help="with the direct transport: push rrc operands into the receiver's FIFO instead of pulling "
                        "them (DESIGN R31)")
    p.add_argument("--nvls", type=int, default=0,
                   help="f3: N>1 only -- send/recv in an NVLS window, NVLS kernel (falls back to --direct if "
                        "the fabric refuses multicast)")
    p.add_argument("--e2e-steps", type=int, default=3)
    p.add_argument("--e2e-check", type=int, default=1, help="compare rank 0's host result with the device run")
    p.add_argument("--inplace-steps", type=int, default=10,
                   help="also time in-place calls (recv = send) -> config.inplace_busbw_gbs")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--tuned-sweep", default="0.0009765625,0.015625,0.0625,0.25,1,4,16,64,256",
                   help="MiB-per-rank sizes for the size-tuned AllReduce (mesh / mesh-port schedules selected "
                        "by minbytes / maxbytes); '' = none")
    p.add_argument("--sweep", default="0.0009765625,1,16,64",
                   help="comma-separated MiB-per-rank sizes for the busBW-vs-size points reported beside the "
                        "headline (slices of the bench buffers; small points are L2-resident); '' = none")
    return p.parse_args()


def load_peaks():
    try:
        with open(PEAKS_FILE) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM, "fallback"


ELT = {"bfloat16": 2, "float16": 2, "float32": 4, "int32": 4}


def ir_text(R, algo: str, n: int, opts: dict) -> str:
    extra = "g=4" if algo == "hm" else ""
    text = R.rescclGenerateIr(algo, "allreduce", n, extra)
    hdr, rest = text.split("\n", 1)
    for k, v in opts.items():
        if v is not None:
            hdr += f" {k}={v}"
    return hdr + "\n" + rest


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q, "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        time.sleep(0.25)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        time.sleep(0.15)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


# ---------------------------------------------------------------------------- CPU oracle leg

def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:  # noqa: BLE001
        return os.cpu_count() or 1


def cpu_oracle_sample(algo: str, n: int, dtype: str, budget_s: float = 12.0):
    """Time the oracle's Python schedule replay (the blocking FIFO simulator, as it
    stands) on a bounded sample of the same workload; returns (busBW-equivalent GB/s,
    seconds per call, sample description)."""
    import resccl_inputs as inp
    from oracle import ir as oir, lower, replay
    g = oir.generate(algo, "allreduce", n, **({"g": 4} if algo == "hm" else {}))
    pl = lower.lower(g)
    count = (4 << 20) // ELT[dtype]          # 4 MiB per rank
    xs = inp.all_inputs(dtype, 0, n, count)
    t0 = time.perf_counter()
    reps = 0
    while True:
        replay.replay(pl, xs, dtype, count, chunk_bytes=1 << 20, instances=1, K=4)
        reps += 1
        if time.perf_counter() - t0 > budget_s:
            break
    dt = (time.perf_counter() - t0) / reps
    S = count * ELT[dtype]
    bus = S / dt * 2 * (n - 1) / n / 1e9
    return bus, dt, f"{algo} allreduce, {n} ranks x {S >> 20} MiB {dtype}, {reps} replay(s), 1 thread (Python)"


def c1_replay_seconds(reps: int = 3) -> float:
    """BASELINE configs[0] -- ring AllReduce of 4096 fp32, 2 ranks, 1 TB, 4 chunks -- as
    the oracle's Python schedule replay: seconds per replay."""
    import resccl_inputs as inp
    from oracle import ir as oir, lower, replay
    g = oir.ring_allreduce(2)
    pl = lower.lower(g)
    xs = inp.all_inputs("float32", 0, 2, 4096)
    t0 = time.perf_counter()
    for _ in range(reps):
        replay.replay(pl, xs, "float32", 4096, chunk_bytes=4096, instances=1, K=4)
    return (time.perf_counter() - t0) / reps


def host_workload(n: int, count: int, dtype: str, seed: int = 0):
    """Synthetic host buffers with the bench workload's shape (uniform [-1, 1), the d2
    value distribution) for the CPU legs."""
    import numpy as np
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(n):
        f = (rng.random(count, dtype=np.float32) * 2 - 1)
        if dtype == "bfloat16":
            out.append((f.view(np.uint32) >> 16).astype(np.uint16))
        elif dtype == "float16":
            out.append(f.astype(np.float16))
        elif dtype == "float32":
            out.append(f)
        else:
            out.append((f * (1 << 20)).astype(np.int32))
    return out


def cpu_fast_replay(algo: str, n: int, dtype: str, xs, count: int, threads: int, reps: int = 1):
    """The oracle's C++ fast replay (oracle/fastreplay.cc) of the WHOLE bench workload;
    returns (busBW-equivalent GB/s, seconds per call)."""
    import numpy as np
    from oracle import fastreplay, ir as oir
    g = oir.generate(algo, "allreduce", n, **({"g": 4} if algo == "hm" else {}))
    outs = [np.empty_like(x) for x in xs]
    fastreplay.replay_full(g, xs, dtype, count, threads=threads, outputs=outs)  # warm (pages, lib load)
    t0 = time.perf_counter()
    for _ in range(reps):
        fastreplay.replay_full(g, xs, dtype, count, threads=threads, outputs=outs)
    dt = (time.perf_counter() - t0) / reps
    S = count * ELT[dtype]
    return S / dt * 2 * (n - 1) / n / 1e9, dt


def cpu_per_config(cores: int, size_mb: int = 64):
    """the oracle's C++ fast replay per BASELINE config family (8 ranks,
    `size_mb` MiB per-rank buffer S, bf16, all host cores): busBW-equivalent GB/s."""
    import numpy as np
    from oracle import fastreplay, ir as oir
    n, e = 8, 2
    out = {}
    for name, coll, kw in (("ring", "allreduce", {}), ("ring", "allgather", {}), ("dbt", "allreduce", {}),
                           ("hm", "allreduce", {"g": 4}), ("synth", "allgather", {"seed": 0, "fanout": 2}),
                           ("synth", "reducescatter", {"seed": 0, "fanout": 2})):
        S = size_mb << 20
        cnt = S // e if coll == "allreduce" else S // e // n      # the collective's count argument
        xs = host_workload(n, cnt * (n if coll == "reducescatter" else 1), "bfloat16", seed=3)
        g = oir.generate(name, coll, n, **kw)
        outs = [np.empty(cnt * (n if coll == "allgather" else 1), np.uint16) for _ in range(n)]
        work = [np.empty(n * cnt, np.uint16) for _ in range(n)] if coll == "reducescatter" else None
        fastreplay.replay_full(g, xs, "bfloat16", cnt, threads=cores, outputs=outs, work=work)  # warm (pages)
        t0 = time.perf_counter()
        fastreplay.replay_full(g, xs, "bfloat16", cnt, threads=cores, outputs=outs, work=work)
        dt = time.perf_counter() - t0
        f = 2 * (n - 1) / n if coll == "allreduce" else (n - 1) / n
        out[f"{name} {coll}"] = round(S / dt / 1e9 * f, 3)
    return out


def reference_impl(args):
    """--impl reference: the oracle timed on the host cores (tier framing).  A step = the
    C++ fast replay of the same workload as the ResCCL arm (same algorithm, ranks, bytes
    per rank, dtype) on every host core."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n = args.vranks if args.gpus == 1 else args.gpus
    count = int(args.size_mb * (1 << 20)) // ELT[args.dtype]
    S = count * ELT[args.dtype]
    cores = host_cores()
    xs = host_workload(n, count, args.dtype)
    for _ in range(args.warmup):
        cpu_fast_replay(args.algo, n, args.dtype, xs, count, cores, reps=1)
    vals, t_all = [], []
    for _ in range(args.steps):
        bus, dt = cpu_fast_replay(args.algo, n, args.dtype, xs, count, cores, reps=1)
        vals.append(bus)
        t_all.append(dt)
    value = S * args.steps / sum(t_all) * 2 * (n - 1) / n / 1e9
    desc = (f"{args.algo} allreduce, {n} ranks x {S >> 20} MiB {args.dtype} (the whole workload), C++ fast "
            f"replay (oracle/fastreplay.cc), {cores} threads")
    line = {
        "impl": "reference", "metric": "allreduce busBW", "value": round(value, 4), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * statistics.mean(t_all), 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": {"bfloat16": "bf16"}.get(args.dtype, args.dtype),
        "data": "synthetic",
        "config": {"workload": f"{args.algo} allreduce, {n} ranks, {S >> 20} MiB per rank, CPU oracle schedule "
                               f"replay on the host cores", "nranks": n, "bytes_per_rank": S},
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------- ResCCL leg

def main():
    args = parse()
    if args.impl == "reference":
        return reference_impl(args)
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("RESCCL_BENCH_ONE_DEVICE") == "1":
        local = 0  # test aid: every rank on cuda:0 (CUDA IPC between processes of one device)
    multi = world > 1
    if multi:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("gloo")
    dev = torch.device("cuda", local if multi else 0)
    n = world if multi else args.vranks
    elt = ELT[args.dtype]
    count = int(args.size_mb * (1 << 20)) // elt
    S = count * elt
    tdt = getattr(torch, args.dtype)
    # Defaults (r01 sweeps, profiles/r01_geo_sweep*.jsonl, profiles/r01_sm_budget_v7.jsonl):
    # the direct transport (R23: push recv payloads, pull rrc operands; no FIFO staging);
    # at N=1 every virtual rank's buffers share one address space, under torchrun (N>1) the
    # send and receive buffers sit in a registered symmetric window.  The lane engine's
    # cost is per TMA tile, so tiles are 24 KiB (2 stages per lane, one CTA per SM):
    #   N=1: 12 instances x 8 virtual ranks = 96 CTAs of 384 threads (65% of the SMs; the
    #        smallest count within 2% of the best busBW, profiles/r02_per_sm_rate.jsonl:
    #        ResCCL's point is fewer TBs), 28 KiB tiles, 32 MiB transfer
    #        chunks (one micro-batch per 32 MiB algorithm chunk);
    #   N>1: 24 CTAs of 384 threads per rank, 28 KiB tiles, 8 MiB chunks.
    direct = 1 if args.direct < 0 else args.direct
    tuned = direct and not args.instances and not args.nwarps
    inst = args.instances or ((12 if not multi else 24) if tuned else 18)
    opts = {"instances": inst,
            "chunkbytes": args.chunk_bytes or ((32 << 20) if (tuned and not multi) else (8 << 20) if direct
                                               else (4 << 20)),
            "fifodepth": args.fifo_depth or 2,
            "nwarps": args.nwarps or ((12 if not multi else 12) if tuned else None),
            "tma": None if args.tma < 0 else args.tma,
            "tmastages": 2 if tuned else None,
            # 28 KiB tiles with 12 warps (384 threads: the register cap of 16 warps, 128 per
            # thread, spills the TMA leader loop): 95-101 GB/s of HBM per SM at 8 CTAs against
            # 85 with 8 warps and 24 KiB tiles (profiles/r02_per_sm_rate.jsonl)
            "tmatile": 28672 if tuned else None,
            "direct": direct, "nvls": 1 if (args.nvls and multi) else None,
            "pushreduce": 1 if (args.pushreduce and direct) else None}
    text = ir_text(R, args.algo, n, opts)

    if multi:
        comm = R.init_process_group_comm(rank, world, local)
        algo = comm.load(text)
        comms = [comm]
    else:
        grp = R.VirtualGroup(n, 0)
        grp.load(text)
        comms = grp.comms
        algo = comms[0].algos[-1]
    info = R.rescclGetPlanInfo(algo)
    blocks = info["blocks_per_rank"]

    gen = torch.Generator(device=dev)
    gen.manual_seed(1234 + rank)
    my_ranks = [rank] if multi else list(range(n))
    sends = {r: (torch.rand(count, generator=gen, device=dev, dtype=torch.float32) * 2 - 1).to(tdt)
             if tdt.is_floating_point else torch.randint(-2 ** 20, 2 ** 20, (count,), device=dev, dtype=tdt)
             for r in my_ranks}
    recvs = {r: torch.empty_like(sends[r]) for r in my_ranks}
    nvls_state = None
    win = None
    if multi and args.nvls:
        from paper_conf_sigcomm_liuhlgcwz025_b200.torch_api import tensor_at
        pad = 256 // elt
        try:
            ptr = comm.nvls_alloc((2 * count + pad) * elt)
            win = tensor_at(ptr, 2 * count + pad, tdt, dev.index)
            win[:count].copy_(sends[rank])
            sends[rank], recvs[rank] = win[:count], win[count + pad:2 * count + pad]
            nvls_state = "nvls window"
        except R.ResCCLError as e:
            nvls_state = f"unavailable ({e}); direct windows used"
    if multi and direct and not (nvls_state or "").startswith("nvls"):
        # symmetric window: [send | pad | recv] at the same offsets on every rank
        pad = 256 // elt
        win = torch.empty(2 * count + pad, dtype=tdt, device=dev)
        win[:count].copy_(sends[rank])
        sends[rank], recvs[rank] = win[:count], win[count + pad:2 * count + pad]
        comm.register(win)
    stream = torch.cuda.current_stream(dev)
    sid = stream.cuda_stream

    def step():
        for r in my_ranks:
            c = comms[0] if multi else comms[r]
            c.allreduce(sends[r], recvs[r], stream=sid)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)

    def barrier():
        if multi:
            torch.distributed.barrier()

    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize(dev)
    with ClockSampler(dev.index) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize(dev)
    barrier()
    ms = ev0.elapsed_time(ev1) / args.steps
    if multi:
        t = torch.tensor([ms], dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    err = comms[0].async_error()
    algbw = S / (ms * 1e-3) / 1e9
    busbw = algbw * 2 * (n - 1) / n

    # ---- end to end: host (pinned) buffers, H2D + collective + D2H inside the timed region
    e2e = None
    if args.e2e_steps > 0:
        hin = {r: sends[r].cpu().pin_memory() for r in my_ranks}
        hout = {r: torch.empty_like(hin[r]).pin_memory() for r in my_ranks}

        def host_step():
            # the C-ABI call on HOST buffers: the library uploads, reduces and downloads
            # (pieces of RESCCL_HOST_PIECE bytes overlapping on two copy streams)
            for r in my_ranks:
                c = comms[0] if multi else comms[r]
                c.allreduce(hin[r], hout[r], stream=sid)

        for _ in range(2):
            host_step()
        torch.cuda.synchronize(dev)
        # pieces reduce in their own chunk order: compare with the device run within the
        # bf16 bound (2e-2 x sum_k |x_k| <= 2e-2 x N for inputs in [-1, 1))
        r0 = my_ranks[0]
        dmax = float((hout[r0].float() - recvs[r0].cpu().float()).abs().max()) if args.e2e_check else None
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            host_step()
        e1.record(stream)
        torch.cuda.synchronize(dev)
        ems = e0.elapsed_time(e1) / args.e2e_steps
        if multi:
            t = torch.tensor([ems], dtype=torch.float64)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            ems = float(t.item())
        e2e_bus = S / (ems * 1e-3) / 1e9 * 2 * (n - 1) / n
        e2e = {"value": round(e2e_bus, 3), "unit": "GB/s", "h2d_bytes_per_step": S * len(my_ranks),
               "d2h_bytes_per_step": S * len(my_ranks), "ms_per_step": round(ems, 3),
               "path": "C-ABI collective on pinned host buffers (library-staged, piecewise H2D/AR/D2H overlap)",
               "piece_bytes": int(os.environ.get("RESCCL_HOST_PIECE", 32 << 20))}
        if dmax is not None:
            e2e["max_abs_diff_vs_device_result"] = dmax
            e2e["within_tolerance"] = bool(dmax <= 2e-2 * n) if tdt.is_floating_point else bool(dmax == 0)

    # ---- in-place (recv = send: the DDP / Megatron bucket case), same workload; the
    # in-place reduce hops take the bulk-reduction path (bulkred, DESIGN 5.4b)
    inplace_bus = None
    if args.inplace_steps > 0:
        def step_inplace():
            for r in my_ranks:
                c = comms[0] if multi else comms[r]
                c.allreduce(sends[r], sends[r], stream=sid)
        for _ in range(2):
            step_inplace()
        torch.cuda.synchronize(dev)
        barrier()
        i0 = torch.cuda.Event(enable_timing=True)
        i1 = torch.cuda.Event(enable_timing=True)
        i0.record(stream)
        for _ in range(args.inplace_steps):
            step_inplace()
        i1.record(stream)
        torch.cuda.synchronize(dev)
        ims = i0.elapsed_time(i1) / args.inplace_steps
        if multi:
            t = torch.tensor([ims], dtype=torch.float64)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            ims = float(t.item())
        inplace_bus = round(S / (ims * 1e-3) / 1e9 * 2 * (n - 1) / n, 2)

    # ---- extra size sweeps (busBW vs size, device clock)
    def graph_sweep(cms, sizes_mb):
        """busBW and time per call for slices of the bench buffers: the calls are captured
        in one CUDA graph (device-side flag epochs) and replayed, so the host's per-call
        submission cost (8 virtual ranks x ctypes + runtime calls, ~60 us) does not hide
        small-message latency."""
        bus, us = {}, {}
        for mb in sizes_mb:
            cnt = int(mb * (1 << 20)) // elt
            if cnt > count:
                continue  # sweep points are slices of the bench buffers
            s2 = {r: sends[r][:cnt] for r in my_ranks}
            r2 = {r: recvs[r][:cnt] for r in my_ranks}
            for _ in range(3):
                for r in my_ranks:
                    (cms[0] if multi else cms[r]).allreduce(s2[r], r2[r], stream=sid)
            torch.cuda.synchronize(dev)
            barrier()
            reps = 10
            cs = torch.cuda.Stream(dev)
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph, stream=cs):
                for _ in range(reps):
                    for r in my_ranks:
                        (cms[0] if multi else cms[r]).allreduce(s2[r], r2[r], stream=cs.cuda_stream)
            graph.replay()
            torch.cuda.synchronize(dev)
            barrier()
            a0 = torch.cuda.Event(enable_timing=True)
            a1 = torch.cuda.Event(enable_timing=True)
            a0.record(cs)
            with torch.cuda.stream(cs):
                graph.replay()
            a1.record(cs)
            torch.cuda.synchronize(dev)
            t_ms = a0.elapsed_time(a1) / reps
            if multi:
                t = torch.tensor([t_ms], dtype=torch.float64)
                torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
                t_ms = float(t.item())
            del graph
            lab = f"{round(mb * 1024)}KiB" if mb < 1 else f"{mb:g}MiB"
            bus[lab] = round(cnt * elt / (t_ms * 1e-3) / 1e9 * 2 * (n - 1) / n, 2)
            us[lab] = round(t_ms * 1e3, 2)
        return bus, us

    sweep, sweep_us = {}, {}
    if args.sweep:
        sweep, sweep_us = graph_sweep(comms, [float(x) for x in args.sweep.split(",") if x])

    # ---- the size-tuned AllReduce (a second communicator set loading several schedules
    # with minbytes / maxbytes ranges, include/resccl.h): the full mesh of Fig. 16 at one
    # node of 8 (HM, nNodes = 1: 7 pull-reduces + 1 push per chunk instead of the ring's 14
    # hops) for small messages, the same mesh under the port link model (one duplex CTA
    # per rank x instances) above 2 MiB.  r02 geometry sweep: profiles/r02_lat_graph_tuned.jsonl
    tuned, tuned_us, tuned_table = {}, {}, None
    if args.tuned_sweep and args.algo == "ring":
        two = 2 << 20
        mesh = f"g={n}"  # the hierarchical mesh at one node of all n ranks: a full mesh
        # r02 late (profiles/r02_lat_classes.jsonl, r02_lat_midgeo.jsonl): the 2x4 hierarchical
        # schedule (HM g=4, pair model, 4 instances) wins from 512 KiB to 8 MiB (1 MiB 52 us,
        # 4 MiB 72 us against the mesh's 56 / 95), 16 mesh instances beat 14 above 32 MiB
        # warp counts (profiles/r02_lat_warps_*.jsonl, r02_lat_ab_classes.jsonl): 18 port-model
        # instances of 128-thread CTAs to 32 MiB (16 MiB 118 us, 32 MiB 182 us on two boxes);
        # above, 16 instances of 256-thread CTAs (the same-box A/B winner at 64 / 256 MiB)
        i_big, i_mid = (16, 18) if not multi else (24, 24)
        w_big, w_mid = (8, 4) if not multi else (8, 8)
        small = 256 << 10
        tuned_table = [("hm", mesh, dict(instances=i_big, chunkbytes=8 << 20, linkmodel="port", nwarps=w_big,
                                         minbytes=(32 << 20) + 1)),
                       ("hm", mesh, dict(instances=i_mid, chunkbytes=8 << 20, linkmodel="port", nwarps=w_mid,
                                         minbytes=(8 << 20) + 1, maxbytes=32 << 20))]
        if n % 4 == 0 and n > 4 and not multi:
            # small messages (profiles/r02_lat_small*.jsonl): 128-thread CTAs; the mesh to 32 KiB
            # (1 KiB 27 us), the 2x4 schedule above (128 KiB 29 us, 1 MiB 49 us)
            small = 32 << 10
            tuned_table.append(("hm", "g=4", dict(instances=4, chunkbytes=512 << 10, nwarps=6, minbytes=two + 1,
                                                  maxbytes=8 << 20)))
            tuned_table.append(("hm", "g=4", dict(instances=4, chunkbytes=512 << 10, nwarps=4, minbytes=small + 1,
                                                  maxbytes=two)))
            tuned_table.append(("hm", mesh, dict(instances=1, chunkbytes=32 << 20, nwarps=4, maxbytes=small)))
        else:  # (N > 1 keeps the round-2 classes: mesh to 2 MiB, mesh under the port model above)
            small = two
            tuned_table[-1][2]["minbytes"] = small + 1
            tuned_table.append(("hm", mesh, dict(instances=2, chunkbytes=two, maxbytes=small)))
        if multi:
            tcomm = R.init_process_group_comm(rank, world, local)
            tcomms = [tcomm]
        else:
            tgrp = R.VirtualGroup(n, 0)
            tcomms = tgrp.comms
        for name, gopt, o in tuned_table:
            t_text = R.rescclGenerateIr(name, "allreduce", n, gopt)
            h2, rest2 = t_text.split("\n", 1)
            h2 += f" nwarps=8 fifodepth=2 direct={direct}" + "".join(f" {k}={v}" for k, v in o.items())
            for c in tcomms:
                c.load(h2 + "\n" + rest2)
        if multi and direct and win is not None and not (nvls_state or "").startswith("nvls"):
            tcomm.register(win)
        tuned, tuned_us = graph_sweep(tcomms, [float(x) for x in args.tuned_sweep.split(",") if x])
        if not multi:
            tgrp.destroy()
        else:
            tcomm.destroy()

    # ---- N > 1 evidence: TB utilisation of one traced call of the same
    # algorithm, and NCCL's AllReduce of the same buffer on the same GPUs -- its busBW and
    # its channel count (NCCL_DEBUG=INFO, one CTA per channel) as the "SMs vs NCCL"
    # denominator.  Every rank runs both (collectives); failures are recorded, not fatal.
    multi_extra = {}
    if multi and args.nccl_compare:
        try:
            tt = R.rescclGenerateIr(args.algo, "allreduce", n, "g=4" if args.algo == "hm" else "")
            h3, rest3 = tt.split("\n", 1)
            h3 += "".join(f" {k}={v}" for k, v in opts.items() if v is not None) + " trace=1"
            ta = comm.load(h3 + "\n" + rest3)
            comm.allreduce(sends[rank], recvs[rank], stream=sid)
            torch.cuda.synchronize(dev)
            u = R.rescclGetTbUtilization(ta)
            multi_extra["tb_utilization"] = {k: round(u[k], 4) if isinstance(u[k], float) else u[k]
                                             for k in ("tbs", "comm_time", "avg_idle", "max_idle", "ctas",
                                                       "cta_comm_time", "cta_avg_idle", "cta_max_idle")}
        except Exception as e:  # noqa: BLE001
            multi_extra["tb_utilization"] = {"error": str(e)[:300]}
        nccl_log = f"/tmp/resccl_bench_nccl.{os.getpid()}.log"
        try:
            import re as _re
            os.environ["NCCL_DEBUG"] = "INFO"
            os.environ["NCCL_DEBUG_SUBSYS"] = "INIT,TUNING"
            os.environ["NCCL_DEBUG_FILE"] = nccl_log
            ng = torch.distributed.new_group(backend="nccl")
            xb = sends[rank].clone()
            for _ in range(3):
                torch.distributed.all_reduce(xb, group=ng)
            torch.cuda.synchronize(dev)
            barrier()
            n0 = torch.cuda.Event(enable_timing=True)
            n1 = torch.cuda.Event(enable_timing=True)
            n0.record()
            for _ in range(10):
                torch.distributed.all_reduce(xb, group=ng)
            n1.record()
            torch.cuda.synchronize(dev)
            nms = n0.elapsed_time(n1) / 10
            t = torch.tensor([nms], dtype=torch.float64)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            nms = float(t.item())
            chan = None
            try:
                txt = open(nccl_log).read()
                m = _re.findall(r"(\d+) coll channels", txt) or _re.findall(r"Channel \d+/(\d+)", txt)
                chan = int(m[-1]) if m else None
            except OSError:
                pass
            multi_extra["nccl"] = {"busbw_gbs": round(S / (nms * 1e-3) / 1e9 * 2 * (n - 1) / n, 2),
                                   "ms": round(nms, 4), "channels": chan,
                                   "ctas_note": "NCCL runs one CTA per channel",
                                   "resccl_ctas_per_rank": blocks[rank]}
        except Exception as e:  # noqa: BLE001
            multi_extra["nccl"] = {"error": str(e)[:300]}

    if rank != 0:
        if multi:
            torch.distributed.destroy_process_group()
        return

    # ---- roofline (dominant and only kernel: the generated schedule kernel)
    peak, peak_src = load_peaks()
    nr = n
    if multi:
        # per GPU: NVLink egress 2(N-1)/N S is the bound (900 GB/s/dir nominal)
        algo_bytes = 2 * (nr - 1) / nr * S
        roof = {"bound": "nvlink", "achieved": round(algo_bytes / (ms * 1e-3) / 1e9, 2), "peak": 900.0,
                "unit": "GB/s", "frac": round(algo_bytes / (ms * 1e-3) / 1e9 / 900.0, 4), "traffic": None,
                "peak_source": "nominal NVLink 5 per direction (measured ref 770 GB/s)"}
    else:
        # Bytes the staged task-level ring AR moves through the memory system per rank
        # (DESIGN.md §5.5): RS hop = send (read s, write FIFO s) + rrc
        # (read FIFO s, read s, write s) = 5s; AG hop = send 2s + recv 2s = 4s; s = S/N
        # => 9(N-1)/N * S.  Every byte crosses the L2 slices (LTS), whose throughput cap is
        # what also bounds the measured HBM copy peak, so that peak is the denominator.
        # dram_algorithmic = the user-buffer share 5(N-1)/N * S (FIFO slots stay in L2).
        # direct transport (R23): no FIFO hop -- RS hop = pull-rrc reads s (peer) + s (own),
        # writes s; AG hop = push-send reads s, writes s (peer) => 5(N-1)/N * S, all HBM.
        per_rank = (5.0 if info.get("direct") else 9.0) * (nr - 1) / nr * S
        algo_bytes = per_rank * nr
        ach = algo_bytes / (ms * 1e-3) / 1e9
        roof = {"bound": "hbm", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
                "frac": round(ach / peak, 4), "traffic": None,
                "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_src}, burst)",
                "algorithmic_bytes_per_launch": int(algo_bytes),
                "dram_algorithmic_bytes_per_launch": int(5.0 * (nr - 1) / nr * S * nr)}
    # measured DRAM traffic of this exact workload from a committed ncu capture (if any)
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            tr = json.load(f)
        key = (f"{args.algo}/{n}/{S}/{args.dtype}/{'direct' if info.get('direct') else 'staged'}/"
               f"{info['instances']}/{info['chunkbytes']}")
        if key in tr:
            roof["traffic"] = tr[key]["traffic"]
            roof["traffic_source"] = tr[key]["source"]
    except Exception:
        pass

    cpu = None
    if not args.no_cpu_baseline and not multi:
        # the oracle as it stands, on the host cores: the C++ fast replay
        # of the whole workload (these very inputs, copied to the host) at all cores and at
        # 1 thread, the Python blocking replay on a bounded sample, and C1 in seconds
        import numpy as np
        xs_host = [(sends[r].cpu().view(torch.int16).numpy().view(np.uint16) if args.dtype == "bfloat16"
                    else sends[r].cpu().numpy()) for r in my_ranks]
        cores = host_cores()
        bus_all, dt_all = cpu_fast_replay(args.algo, n, args.dtype, xs_host, count, cores, reps=2)
        bus_1, dt_1 = cpu_fast_replay(args.algo, n, args.dtype, xs_host, count, 1, reps=1)
        del xs_host
        bus_py, dt_py, desc_py = cpu_oracle_sample(args.algo, n, args.dtype, budget_s=6.0)
        cpu = {"value": round(bus_all, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
               "sample": (f"the whole workload ({n} ranks x {S >> 20} MiB {args.dtype}, this run's inputs): "
                          f"C++ fast replay (oracle/fastreplay.cc), {cores} threads, 2 calls"),
               "s_per_call": round(dt_all, 3),
               "one_thread": {"value": round(bus_1, 4), "unit": "GB/s", "cores": 1, "s_per_call": round(dt_1, 3)},
               "python_replay": {"value": round(bus_py, 4), "unit": "GB/s", "cores": 1,
                                 "s_per_call": round(dt_py, 3), "sample": desc_py},
               "c1_replay_s": round(c1_replay_seconds(), 4),
               "per_config_64MiB": cpu_per_config(cores),
               "c1": "BASELINE configs[0]: ring AllReduce 4096 fp32, 2 ranks, 1 TB, 4 chunks (Python replay)"}

    # SMs the kernel occupies: its CTAs (one or two per SM, by block size) spread over the SMs
    n_sm = torch.cuda.get_device_properties(dev).multi_processor_count
    sms = min(n_sm, sum(blocks) if not multi else blocks[rank])
    if (nvls_state or "").startswith("nvls"):
        sms = min(n_sm, info.get("nvlsctas", 16))  # upper bound: the grid shrinks for small messages
    line = {
        "metric": "allreduce busBW", "value": round(busbw, 2), "unit": "GB/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None,
        "dtype": {"bfloat16": "bf16", "float16": "f16", "float32": "f32", "int32": "i32"}[args.dtype],
        "data": "synthetic",
        "config": {
            "workload": (f"{args.algo} allreduce, {n} virtual ranks on 1 B200 (all ranks' buffers and FIFOs "
                         f"in one HBM), {S >> 20} MiB per rank" if not multi else
                         f"{args.algo} allreduce, {n} GPUs (CUDA-IPC NVLink), {S >> 20} MiB per rank"),
            "nranks": n, "bytes_per_rank": S, "algo": args.algo, "instances": info["instances"],
            "chunkbytes": info["chunkbytes"], "fifodepth": info["fifodepth"], "nwarps": info["nwarps"],
            "linkmodel": info["linkmodel"], "transport": ("nvls" if (nvls_state or "").startswith("nvls") else
                                                   "direct" if info.get("direct") else "staged-fifo"),
            **({"nvls": nvls_state} if nvls_state else {}),
            "ctas_per_rank": info["ctas"], "blocks_total": sum(blocks),
            "sms_used": sms, "algbw_gbs": round(algbw, 2), "inplace_busbw_gbs": inplace_bus, "l2": "inputs > L2 on every rank (no flush)",
            "parallelism": "virtual-ranks" if not multi else f"ranks{n}",
        },
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": args.steps * (1 if not multi else 1),
        "clocks": clk.summary(),
        "async_error": err,
    }
    if sweep:
        line["sweep_busbw_gbs"] = sweep  # busBW vs size (BASELINE metric); not the headline value
        line["sweep_us"] = sweep_us      # device-clock time per call (CUDA-graph replay)
        line["sweep_timing"] = "CUDA-graph replay of 10 calls (device clock; host submission excluded)"
    if multi_extra:
        line["multi_gpu"] = multi_extra
    if tuned:
        line["tuned_busbw_gbs"] = tuned  # size-tuned schedule selection (mesh / mesh-port)
        line["tuned_us"] = tuned_us
        line["tuned_schedules"] = [f"{a} {g} " + " ".join(f"{k}={v}" for k, v in o.items()) for a, g, o in tuned_table]
    print(json.dumps(line), flush=True)
    if multi:
        torch.distributed.destroy_process_group()
    else:
        grp.destroy()


if __name__ == "__main__":
    main()
