"""Table 3 analogue on one B200: TB count and TB utilisation (Comm Time / Avg Idle /
Max Idle) per schedule, measured with RESCCL_TRACE lane timers on 8
virtual ranks.  Usage: python tools/tb_util.py [size_mb] [geo]
  geo = r01 (instances=2, 1 MiB chunks, staged FIFO: the round-1 table) or
        best (each schedule's best geometry of profiles/r02_geo_trees.jsonl, direct)"""
import json
import sys
import os

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigcomm_liuhlgcwz025_b200 as R

size_mb = float(sys.argv[1]) if len(sys.argv) > 1 else 64
geo = sys.argv[2] if len(sys.argv) > 2 else "r01"
BEST = {  # (name, coll) -> geometry (r02 geometry sweep, 256 MiB, direct transport)
    ("ring", "allreduce"): "instances=14 chunkbytes=33554432 nwarps=8 direct=1",
    ("ring", "allgather"): "instances=18 chunkbytes=8388608 nwarps=8 direct=1",
    ("dbt", "allreduce"): "instances=6 chunkbytes=8388608 nwarps=8 direct=1",
    ("hm", "allreduce"): "instances=4 chunkbytes=1048576 nwarps=8 direct=1",
    ("hm", "allgather"): "instances=4 chunkbytes=4194304 nwarps=8 direct=1",
    ("synth", "allgather"): "instances=4 chunkbytes=8388608 nwarps=8 direct=1",
    ("synth", "reducescatter"): "instances=4 chunkbytes=1048576 nwarps=8 direct=1",
}
cases = [
    ("ring", "allreduce", "", ""), ("dbt", "allreduce", "", ""), ("hm", "allreduce", "g=4", ""),
    ("hm", "allgather", "g=4", ""), ("ring", "allgather", "", ""),
    ("synth", "allgather", "seed=0 fanout=2", ""), ("synth", "reducescatter", "seed=1 fanout=3", ""),
    ("hm", "allreduce", "g=4", "linkmodel=port"), ("dbt", "allreduce", "", "linkmodel=port"),
]
out = []
for name, coll, gopts, popts in cases:
    n = 8
    text = R.rescclGenerateIr(name, coll, n, gopts)
    hdr, rest = text.split("\n", 1)
    g = BEST[(name, coll)] if geo == "best" else "instances=2 chunkbytes=1048576"
    text = hdr + f" {g} fifodepth=2 trace=1 {popts}\n" + rest
    grp = R.VirtualGroup(n, 0)
    grp.load(text)
    info = grp.plan_info()
    cnt = int(size_mb * (1 << 20)) // 2
    send_n = cnt * n if coll == "reducescatter" else cnt
    recv_n = cnt * n if coll == "allgather" else cnt
    s = [torch.randn(send_n, device="cuda:0").to(torch.bfloat16) for _ in range(n)]
    r = [torch.empty(recv_n, device="cuda:0", dtype=torch.bfloat16) for _ in range(n)]
    for _ in range(3):
        getattr(grp, coll)(s, r)
    torch.cuda.synchronize()
    u = R.rescclGetTbUtilization(grp.comms[0].algos[-1])
    paper_tbs = [rk["paper_tbs"] for rk in info["plan"]["ranks"]]
    row = {"algo": f"{name} {coll} {gopts} {popts}".strip(), "geometry": g, "bytes": int(size_mb * (1 << 20)),
           "ctas_per_rank": info["ctas"],
           "paper_tbs_per_rank": paper_tbs, "n_connections": [rk["n_connections"] for rk in info["plan"]["ranks"]],
           "instances": info["instances"], "traced_lanes": u["tbs"], "comm_time": round(u["comm_time"], 4),
           "avg_idle": round(u["avg_idle"], 4), "max_idle": round(u["max_idle"], 4),
           "span_us": round(u["span_ns"] / 1e3, 1), "fused": info["plan"]["fused"],
           # per CTA (= one SM): fraction of its lifetime with both lanes busy-waiting / done
           "ctas": u["ctas"], "cta_comm_time": round(u["cta_comm_time"], 4),
           "cta_avg_idle": round(u["cta_avg_idle"], 4), "cta_max_idle": round(u["cta_max_idle"], 4)}
    out.append(row)
    print(json.dumps(row), flush=True)
    grp.destroy()
