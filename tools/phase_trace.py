"""Phase breakdown of one collective launch.

Loads the algorithm with phase=1 (every lane leader stamps %globaltimer per primitive and
micro-batch, include/resccl.h rescclGetPhaseTrace), runs a few warm-up calls and one
traced call, then walks the critical path backwards from the last post using the plan's
own producer relation (local counters, the sender of a payload / readable flag, the
receiver of a writable credit).  Every link of the path is split into

  handoff : producer's post -> consumer saw it (flag trip through L2 + polling)
  wait    : consumer was not yet waiting (it was busy with an earlier primitive)
  data    : flag seen -> data moved (register path) or stores complete (TMA engine)
  post    : fence + flag / counter stores

Usage: python tools/phase_trace.py [sizes in bytes ...]   (env PHASE_OPTS, PHASE_N)
Prints one JSON line per size."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_sigcomm_liuhlgcwz025_b200 as R  # noqa: E402

N = int(os.environ.get("PHASE_N", "8"))
ALGO = os.environ.get("PHASE_ALGO", "ring")
GOPTS = os.environ.get("PHASE_GOPTS", "g=4" if ALGO == "hm" else "")
OPTS = os.environ.get("PHASE_OPTS", "instances=14 nwarps=8 chunkbytes=33554432 fifodepth=2 direct=1")


def decode(words):
    blocks, base, P, inst = words[:4]
    lanes = []
    for b in range(blocks):
        for ln in range(2):
            off = 4 + (2 * b + ln) * 8 * P
            hdr = words[off:off + 8]
            if hdr[0] == 0:
                continue
            recs = []
            for k in range(1, int(hdr[2]) + 1):
                r = words[off + 8 * k: off + 8 * k + 8]
                recs.append({"prim": r[0] >> 32, "mb": (r[0] >> 8) & 0xFFFFFF, "kind": r[0] & 0xFF,
                             "t": list(r[1:6]), "tc": r[6], "d_run": r[7] & 0xFFFF, "d_pro": (r[7] >> 16) & 0xFFFF,
                             "d_ret": (r[7] >> 32) & 0xFFFF})
            lanes.append({"block": b, "lane": ln, "entry": hdr[0], "exit": hdr[1], "rank": hdr[3],
                          "cta": hdr[4], "inst": hdr[5], "recs": recs})
    return lanes


def ready_time(rec):
    t = rec["t"]
    if rec["kind"] == 0:
        return t[2]          # flag / credit met
    if rec["kind"] == 1:
        return t[2] or t[1]  # payload seen (push receive) or dependencies met
    return t[1]              # TMA engine: ready


def analyse(lanes, plan, inst=0):
    ranks = plan["ranks"]
    tasks = plan["tasks"]
    by = {}
    for L in lanes:
        if L["inst"] != inst:
            continue
        for rec in L["recs"]:
            by[(L["rank"], rec["prim"], rec["mb"])] = (rec, L)
    send_of, recv_of = {}, {}
    for r, rp in enumerate(ranks):
        for k, pm in enumerate(rp["prims"]):
            if pm["send_task"] >= 0:
                send_of[pm["send_task"]] = (r, k)
            if pm["recv_task"] >= 0:
                recv_of[pm["recv_task"]] = (r, k)

    def producers(r, k, j):
        pm = ranks[r]["prims"][k]
        out = [(r, d, j) for d in pm["deps"] + pm["ack_deps"]]
        if pm["recv_task"] >= 0 and pm["recv_task"] in send_of:
            out.append(send_of[pm["recv_task"]] + (j,))
        if pm["send_task"] >= 0 and pm["kind"] in ("dsend", "drecv_d") and pm["send_task"] in recv_of:
            out.append(recv_of[pm["send_task"]] + (j,))          # "writable" credit
        return [x for x in out if x in by]

    last = max(by, key=lambda x: by[x][0]["t"][4])
    t_first = min(L["entry"] for L in lanes)
    t0_all = t_first
    t_last = max(L["exit"] for L in lanes)
    path = []
    cur = last
    seen = set()
    while cur and cur not in seen:
        seen.add(cur)
        rec, L = by[cur]
        prods = producers(*cur)
        rdy = ready_time(rec)
        best = None
        for pkey in prods:
            prec = by[pkey][0]
            if prec["t"][4] and prec["t"][4] <= rec["t"][4] and (best is None or prec["t"][4] > by[best][0]["t"][4]):
                best = pkey
        start = rec["t"][0]
        link = {"rank": cur[0], "prim": ranks[cur[0]]["prims"][cur[1]]["kind"], "chunk": ranks[cur[0]]["prims"][cur[1]]["chunk"],
                "mb": cur[2], "data_ns": (rec["t"][3] - rdy) if rec["t"][3] and rdy else 0,
                "post_ns": rec["t"][4] - (rec["t"][3] or rdy or rec["t"][4]),
                "t_rel_ns": [(x - t0_all) if x else None for x in rec["t"]],
                "producers": [{"rank": pk[0], "prim": ranks[pk[0]]["prims"][pk[1]]["kind"],
                               "post_rel_ns": by[pk][0]["t"][4] - t0_all} for pk in prods]}
        if best is not None:
            ppost = by[best][0]["t"][4]
            link["handoff_ns"] = max(0, rdy - max(ppost, start)) if rdy else 0
            link["wait_ns"] = max(0, start - ppost)
        else:
            link["handoff_ns"] = 0
            link["from_entry_ns"] = (rdy or rec["t"][4]) - L["entry"]
        path.append(link)
        cur = best
    path.reverse()
    tot = {k: sum(p.get(k, 0) for p in path) for k in ("handoff_ns", "wait_ns", "data_ns", "post_ns")}
    return {"span_ns": t_last - t_first, "path_links": len(path), "totals": tot,
            "first_entry_to_first_ready_ns": path[0].get("from_entry_ns", 0) if path else 0,
            "entry_skew_ns": max(L["entry"] for L in lanes) - t_first,
            "exit_after_last_post_ns": t_last - by[last][0]["t"][4],
            "path": path}


def per_kind(lanes, plan):
    out = {}
    for L in lanes:
        for rec in L["recs"]:
            kind = plan["ranks"][L["rank"]]["prims"][rec["prim"]]["kind"]
            t = rec["t"]
            rdy = ready_time(rec)
            d = out.setdefault(kind, {"post": [], "data": []})
            d["post"].append(t[4] - (t[3] or rdy or t[4]))
            if t[3] and rdy:
                d["data"].append(t[3] - rdy)
    return {k: {"n": len(v["post"]), "post_med_ns": statistics.median(v["post"]) if v["post"] else None,
                "data_med_ns": statistics.median(v["data"]) if v["data"] else None} for k, v in out.items()}


def _graph_us(grp, s, r):
    import torch
    st = torch.cuda.Stream()
    gph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gph, stream=st):
        grp.allreduce(s, r, stream=st)
    for _ in range(3):
        gph.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        gph.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / 20


def main():
    sizes = [int(x) for x in sys.argv[1:]] or [1024, 1 << 20, 16 << 20]
    text = R.rescclGenerateIr(ALGO, "allreduce", N, GOPTS)
    hdr, rest = text.split("\n", 1)
    for S in sizes:
        grp = R.VirtualGroup(N, 0)
        try:
            grp.load(hdr + " " + OPTS + " phase=1\n" + rest)
            cnt = S // 2
            s = [torch.randn(cnt, device="cuda:0").to(torch.bfloat16) for _ in range(N)]
            r = [torch.empty_like(x) for x in s]
            for _ in range(5):
                grp.allreduce(s, r)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            # (a) back-to-back eager calls: max(host submit, GPU) per call
            import time as _t
            h0 = _t.perf_counter()
            e0.record()
            for _ in range(20):
                grp.allreduce(s, r)
            e1.record()
            host_us = (_t.perf_counter() - h0) / 20 * 1e6
            torch.cuda.synchronize()
            loop_us = e0.elapsed_time(e1) * 1e3 / 20
            # (b) the same call captured in a CUDA graph: GPU time per call (needs device-side
            # epochs: PHASE_NOGRAPH=1 skips it for devepoch=0 runs)
            if os.environ.get("PHASE_NOGRAPH") == "1":
                graph_us = float("nan")
            else:
                graph_us = _graph_us(grp, s, r)
            # (c) one traced call (the analysed one)
            e0.record()
            grp.allreduce(s, r)
            e1.record()
            torch.cuda.synchronize()
            us = e0.elapsed_time(e1) * 1e3
            algo = grp.comms[0].algos[-1]
            plan = R.rescclGetPlanInfo(algo)["plan"]
            lanes = decode(R.rescclGetPhaseTrace(algo))
            a = analyse(lanes, plan)
            out = {"bytes": S, "opts": OPTS, "algo": ALGO, "n": N, "event_us": round(us, 2),
                   "eager_loop_us": round(loop_us, 2), "host_submit_us": round(host_us, 2),
                   "graph_replay_us": round(graph_us, 2),
                   "span_us": round(a["span_ns"] / 1e3, 2), "launch_overhead_us": round(us - a["span_ns"] / 1e3, 2),
                   "critical_path": {k: round(v / 1e3, 2) for k, v in a["totals"].items()},
                   "path_links": a["path_links"], "entry_skew_us": round(a["entry_skew_ns"] / 1e3, 2),
                   "first_ready_after_entry_us": round(a["first_entry_to_first_ready_ns"] / 1e3, 2),
                   "exit_after_last_post_us": round(a["exit_after_last_post_ns"] / 1e3, 2),
                   "per_kind": per_kind(lanes, plan), "path": a["path"]}
            print(json.dumps(out), flush=True)
            if os.environ.get("PHASE_RAW"):  # every lane of instance 0, for offline timelines
                kinds = [[pm["kind"] for pm in rp["prims"]] for rp in plan["ranks"]]
                with open(os.environ["PHASE_RAW"], "a") as f:
                    f.write(json.dumps({"bytes": S, "opts": OPTS, "algo": ALGO, "kinds": kinds,
                                        "lanes": [L for L in lanes if L["inst"] == 0]}) + "\n")
        finally:
            grp.destroy()


if __name__ == "__main__":
    main()
