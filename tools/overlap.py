"""Config C5 analogue on one B200: a bf16 GEMM loop on one stream, 25 MiB bf16 bucket
AllReduces (ring, 8 virtual ranks, direct transport) on another; GEMM TFLOP/s alone vs
concurrent, and AR time, for several SM budgets (instances -> 8 x instances CTAs)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
M = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
ALGO = os.environ.get("OVERLAP_ALGO", "ring")
GOPTS = os.environ.get("OVERLAP_GOPTS", "")
OPTS = os.environ.get("OVERLAP_OPTS", "chunkbytes=4194304 direct=1")
INSTS = [int(x) for x in os.environ.get("OVERLAP_INSTANCES", "1,2,4,8,18").split(",")]
a = torch.randn(M, M, device="cuda:0", dtype=torch.bfloat16)
b = torch.randn(M, M, device="cuda:0", dtype=torch.bfloat16)
c = torch.empty(M, M, device="cuda:0", dtype=torch.bfloat16)
sg = torch.cuda.Stream()
sc = torch.cuda.Stream()
flops = 2 * M ** 3


def gemm_loop(n):
    with torch.cuda.stream(sg):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(sg)
        for _ in range(n):
            torch.matmul(a, b, out=c)
        e1.record(sg)
    return e0, e1


def gemm_alone():
    e0, e1 = gemm_loop(40)
    torch.cuda.synchronize()
    return flops * 40 / (e0.elapsed_time(e1) * 1e-3) / 1e12


# warm the GPU to its steady clock first (a cold first measurement made GEMM-alone look slow
# and the concurrent run "faster"), then pair every concurrent run with its own GEMM-alone run
for _ in range(150):
    torch.matmul(a, b, out=c)
torch.cuda.synchronize()
alone = gemm_alone()
print(json.dumps({"gemm_alone_tflops": round(alone, 1), "M": M}), flush=True)

cnt = 25 * (1 << 20) // 2
for inst in INSTS:
    text = R.rescclGenerateIr(ALGO, "allreduce", N, GOPTS)
    h, rest = text.split("\n", 1)
    grp = R.VirtualGroup(N, 0)
    grp.load(h + f" instances={inst} {OPTS}\n" + rest)
    info = grp.plan_info()
    s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
    r = [torch.empty_like(x) for x in s]
    for _ in range(3):
        grp.allreduce(s, r, stream=sc.cuda_stream)
    torch.cuda.synchronize()
    # AR alone
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(sc)
    for _ in range(40):
        grp.allreduce(s, r, stream=sc.cuda_stream)
    f1.record(sc)
    torch.cuda.synchronize()
    ar_alone = f0.elapsed_time(f1) / 40
    alone = gemm_alone()  # paired: right before the concurrent run
    # concurrent
    g0, g1 = gemm_loop(40)
    f0.record(sc)
    for _ in range(40):
        grp.allreduce(s, r, stream=sc.cuda_stream)
    f1.record(sc)
    torch.cuda.synchronize()
    conc = flops * 40 / (g0.elapsed_time(g1) * 1e-3) / 1e12
    ar_conc = f0.elapsed_time(f1) / 40
    print(json.dumps({"algo": ALGO, "gopts": GOPTS, "opts": OPTS, "instances": inst,
                      "comm_ctas": sum(info["blocks_per_rank"]), "gemm_concurrent_tflops": round(conc, 1),
                      "gemm_alone_tflops": round(alone, 1), "gemm_slowdown_pct": round(100 * (1 - conc / alone), 2), "ar_alone_us": round(ar_alone * 1e3, 1),
                      "ar_concurrent_us": round(ar_conc * 1e3, 1), "bucket_mib": 25,
                      "err": grp.async_error()}), flush=True)
    grp.destroy()
