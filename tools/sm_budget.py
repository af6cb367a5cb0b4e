"""SMs used vs bandwidth (the Fig. 4 analogue on one B200): ring AllReduce,
8 virtual ranks, bf16, S MiB per rank, direct transport, for a range of instance counts
(CTAs per rank).  One JSON line per point: busBW, HBM rate (5(N-1)/N * S * N algorithmic
bytes) and the SMs the launch occupies.

  python tools/sm_budget.py [S_MiB] [geometry ...]
geometry: "two" = 256-thread CTAs, 2 x 12 KiB-tile stages (two CTAs per SM);
          "one" = 512-thread CTAs, 4 x 12 KiB-tile stages (one CTA per SM)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

N = 8
S = int(float(sys.argv[1]) * (1 << 20)) if len(sys.argv) > 1 else 256 << 20
GEOS = sys.argv[2:] or ["two", "one"]
GEO = {"two": dict(nwarps=8, tmastages=2, tmatile=12288), "one": dict(nwarps=16, tmastages=4, tmatile=12288)}
for g in GEOS:  # "w<nwarps>s<stages>t<tile>", e.g. w16s8t6144
    if g.startswith("w") and "s" in g and "t" in g:
        w, rest = g[1:].split("s")
        st, t = rest.split("t")
        GEO[g] = dict(nwarps=int(w), tmastages=int(st), tmatile=int(t))
EXTRA = os.environ.get("SMB_OPTS", "")
COLL = os.environ.get("SMB_COLL", "allreduce")
INST = [int(x) for x in os.environ.get("SMB_INST", "1,2,3,4,6,8,10,12,16,18,24,30,37").split(",")]
n_sm = torch.cuda.get_device_properties(0).multi_processor_count

cnt = S // 2  # AR: count; AG: total output; RS: total input (nccl-tests S)
sn, rn = {"allreduce": (cnt, cnt), "allgather": (cnt // N, cnt), "reducescatter": (cnt, cnt // N)}[COLL]
s = [(torch.rand(sn, device="cuda:0") * 2 - 1).to(torch.bfloat16) for _ in range(N)]
r = [torch.empty(rn, device="cuda:0", dtype=torch.bfloat16) for _ in range(N)]
if os.environ.get("SMB_INPLACE") == "1":  # in-place (AllReduce: recv = send; RS: recv inside send)
    r = [s[k] if COLL == "allreduce" else s[k][k * rn:(k + 1) * rn] for k in range(N)]
# algorithmic HBM bytes per rank (direct transport): AR 5(N-1)/N S, RS 3(N-1)/N S, AG 2(N-1)/N S
HB = {"allreduce": 5.0, "reducescatter": 3.0, "allgather": 2.0}[COLL]
BUSF = {"allreduce": 2.0 * (N - 1) / N}.get(COLL, (N - 1) / N)
for geo in GEOS:
    for inst in INST:
        if geo != "two" and inst * N > n_sm:
            continue
        if inst * N > 2 * n_sm:
            continue
        cb = int(os.environ.get("SMB_CB", max(1 << 20, min(32 << 20, S // N))))
        opts = dict(instances=inst, chunkbytes=cb, fifodepth=2, direct=1, **GEO[geo])
        text = R.rescclGenerateIr("ring", COLL, N)
        h, rest = text.split("\n", 1)
        h += "".join(f" {k}={v}" for k, v in opts.items()) + (" " + EXTRA if EXTRA else "")
        grp = R.VirtualGroup(N, 0)
        try:
            grp.load(h + "\n" + rest)
            info = grp.plan_info()
            for _ in range(3):
                getattr(grp, COLL)(s, r)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            it = 10
            e0.record()
            for _ in range(it):
                getattr(grp, COLL)(s, r)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / it
            blocks = sum(info["blocks_per_rank"])
            bus = S / (ms * 1e-3) / 1e9 * BUSF
            hbm = HB * (N - 1) / N * S * N / (ms * 1e-3) / 1e9
            print(json.dumps({"coll": COLL, "geometry": geo, "instances": inst, "ctas": blocks,
                              "sms": min(n_sm, blocks),
                              "S": S, "us": round(ms * 1e3, 1), "busbw_gbs": round(bus, 1),
                              "hbm_gbs": round(hbm, 1), "per_sm_hbm_gbs": round(hbm / min(n_sm, blocks), 1),
                              "opts": EXTRA, "inplace": os.environ.get("SMB_INPLACE") == "1",
                              "err": grp.async_error()}), flush=True)
        finally:
            grp.destroy()
