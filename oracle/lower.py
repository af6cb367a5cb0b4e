"""Oracle: task->primitive translation, state-based TB allocation and fusion.
TEST INFRASTRUCTURE ONLY.

* Translation (Fig. 5e "Transfer = Sender + Receiver"): task t
  becomes send(t) on t.src and recv(t) / rrc(t) on t.dst; both carry t's
  pipeline index (the index of its sub-pipeline Pc in Pr).
* Connection-based allocation: one TB per connection, |C|.
* State-based allocation (Eq. 7): a connection of rank r is
  (peer, send|recv); its activity is the set of pipeline indices where it has a
  primitive (reading R15).  Connections whose activities are disjoint are merged
  ("never active simultaneously").  Merging is greedy colouring, per direction,
  over connections sorted by (first active index, peer): each joins the first
  group it is disjoint with, else opens a new group.  Send group i and recv group
  i form CTA i (a send lane and a recv lane of independent warps, reading R20),
  so #CTA = max(#send groups, #recv groups); the paper-parity TB count (R14)
  is #send groups + #recv groups.
* Local dependencies: DAG edge u->v induced at rank x becomes "prim(u@x)
  precedes prim(v@x)" for every micro-batch (rule (1)).  A dependency
  between two primitives of one lane is implied by the lane's pipeline order (the
  task-level constraint) and needs no counter.
* Fusion (the north_star's recvReduceSend / recvCopySend): on
  rank r, recv-lane primitive a = recv/rrc(t1) of CTA i absorbs send primitive
  b = send(t2) of the same CTA's send lane when b's only local dependency is a.
  The fused primitive stores the received value locally unless the value is read
  by nobody but t2 and is later overwritten (or is not an output).  Candidates are
  tried in lane order; a takes the eligible b with the smallest (pipeline index,
  dst).  Fusion is dropped for the whole plan if it makes the plan deadlock.
* Buffer mapping (R18, in-place IR, out-of-place execution): a read of <r,c>
  before the first write of <r,c> reads the caller's send buffer; later reads and
  all writes use the receive buffer, except ReduceScatter chunks c != r, which
  live in a comm-owned scratch buffer.  An output location never written on r
  (AllGather's own chunk) is stored locally by the first send that moves it out of the
  send buffer (``store`` on a send / dsend: one read feeds the peer and the local copy);
  only when no such send exists (N = 1) does it get a copy primitive at the head of
  CTA 0's recv lane.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Tuple

from .dag import build_dag, check_defined_reads, accesses
from .hpds import hpds, pipeline_index
from .ir import IR, RRC


@dataclass
class Prim:
    rank: int
    kind: str                 # send recv rrc copy rrs rrcs rcs rs
    chunk: int
    pc: int
    recv_task: Optional[int] = None   # task whose payload this prim consumes
    send_task: Optional[int] = None   # task whose payload this prim produces
    reduce: bool = False
    store: bool = False
    src_buf: Optional[str] = None     # local operand: send | recv | scratch
    dst_buf: Optional[str] = None     # local store target: recv | scratch
    cta: int = 0
    lane: str = "S"                   # S (send lane) | R (recv lane)
    deps: List[int] = field(default_factory=list)   # prim ids (same rank) waited on
    ack_deps: List[int] = field(default_factory=list)  # direct: pull-sends completed by the peer's ack
    direct: bool = False
    pull: bool = False
    rem_buf: Optional[str] = None     # direct: buffer of the peer location a pull reads
    rem_out: Optional[str] = None     # direct: buffer of the peer location a push writes
    has_counter: bool = False
    pid: int = -1

    def key(self, tasks):
        """Hashable description used to compare plans between implementations."""
        rt = tuple(tasks[self.recv_task]) if self.recv_task is not None else None
        st = tuple(tasks[self.send_task]) if self.send_task is not None else None
        return (self.kind, self.chunk, self.pc, rt, st, self.src_buf, self.dst_buf)


DIRECT_FUSED = {("prrc", "psend"): "prrc_p", ("prrc", "dsend"): "prrc_d",
                ("drecv", "psend"): "drecv_p", ("drecv", "dsend"): "drecv_d"}
PULL_SENDS = ("psend", "prrc_p", "drecv_p")      # outgoing task pulled: post "readable" only
PUSH_RECVS = ("drecv", "drecv_p", "drecv_d")     # incoming payload pushed into our location


FUSED_KIND = {  # (recv op, store) -> fused name
    ("rrc", False): "rrs", ("rrc", True): "rrcs",
    ("recv", True): "rcs", ("recv", False): "rs",
}


@dataclass
class Plan:
    ir: IR
    model: str
    edges: list
    edge_rank: dict
    Pr: List[List[int]]
    pidx: List[int]
    prims: Dict[int, List[Prim]]                  # rank -> prims (pid = index)
    lanes: Dict[int, List[Tuple[List[int], List[int]]]]   # rank -> [(send pids, recv pids)] per CTA
    send_groups: Dict[int, List[List[Tuple[int, str]]]]
    recv_groups: Dict[int, List[List[Tuple[int, str]]]]
    n_connections: Dict[int, int]
    fused: bool
    direct: bool = False

    def ctas(self, r: int) -> int:
        return len(self.lanes[r])

    def paper_tbs(self, r: int) -> int:
        return len(self.send_groups[r]) + len(self.recv_groups[r])

    def clique_bound(self, r: int) -> Tuple[int, int]:
        """max over pipeline indices of #active send / recv connections (I5)."""
        best = [0, 0]
        for k in range(len(self.Pr)):
            for d, groups in enumerate((self.send_groups[r], self.recv_groups[r])):
                n = 0
                for g in groups:
                    for conn in g:
                        if k in self._act[r][conn]:
                            n += 1
                best[d] = max(best[d], n)
        return best[0], best[1]


def is_output(coll: str, r: int, c: int) -> bool:
    return coll != "reducescatter" or c == r


def write_buf(coll: str, r: int, c: int) -> str:
    return "scratch" if (coll == "reducescatter" and c != r) else "recv"


def _greedy_merge(conns_act: Dict[Tuple[int, str], set]) -> List[List[Tuple[int, str]]]:
    order = sorted(conns_act, key=lambda cn: (min(conns_act[cn]), cn[0]))
    groups: List[List[Tuple[int, str]]] = []
    gact: List[set] = []
    for cn in order:
        for gi, ga in enumerate(gact):
            if not (ga & conns_act[cn]):
                groups[gi].append(cn)
                ga |= conns_act[cn]
                break
        else:
            groups.append([cn])
            gact.append(set(conns_act[cn]))
    return groups


def lower(ir: IR, model: str = "pair", fuse: bool = True, Pr=None, direct: bool = False,
          pushreduce: bool = False) -> Plan:
    """``direct`` (reading R23): no FIFO staging; recv tasks are pushed into the
    receiver's location after it posts "writable", rrc tasks are pulled from the
    sender's location, whose completion is the receiver's read acknowledgement.
    Fusion in direct mode chains a receive with the next hop's push or "readable".
    ``pushreduce`` (with ``direct``, DESIGN R31): rrc tasks keep the staged FIFO (the
    sender pushes its operand into the receiver's slot, the receiver reduces locally);
    recv tasks stay direct pushes.  Only primitives of the same mode fuse."""
    edges, edge_rank = build_dag(ir)
    check_defined_reads(ir)
    if Pr is None:
        Pr = hpds(ir, edges, model)
    tasks = ir.transfers
    nt = len(tasks)
    pidx = pipeline_index(Pr, nt)
    N = ir.nranks
    coll = ir.coll

    # -- first write step of every location (for the send-buffer / receive-buffer choice)
    first_w: Dict[Tuple[int, int], int] = {}
    loc_acc: Dict[Tuple[int, int], List[Tuple[int, int, str]]] = {}
    for i, t in enumerate(tasks):
        for loc, kind in accesses(t):
            loc_acc.setdefault(loc, []).append((t.step, i, kind))
            if kind != "R":
                first_w[loc] = min(first_w.get(loc, 1 << 60), t.step)
    for loc in loc_acc:
        loc_acc[loc].sort()

    def read_buf(r, c, step):
        if (r, c) in first_w and first_w[(r, c)] < step:
            return write_buf(coll, r, c)
        return "send"

    # -- translation
    prims: Dict[int, List[Prim]] = {r: [] for r in range(N)}
    send_of: Dict[int, Tuple[int, int]] = {}
    recv_of: Dict[int, Tuple[int, int]] = {}
    for i, t in enumerate(tasks):
        s = Prim(t.src, "send", t.chunk, pidx[i], send_task=i,
                 src_buf=read_buf(t.src, t.chunk, t.step))
        s.pid = len(prims[t.src]); prims[t.src].append(s); send_of[i] = (t.src, s.pid)
        rv = Prim(t.dst, t.op, t.chunk, pidx[i], recv_task=i, reduce=(t.op == RRC),
                  store=True, dst_buf=write_buf(coll, t.dst, t.chunk),
                  src_buf=read_buf(t.dst, t.chunk, t.step) if t.op == RRC else None)
        if direct:
            if t.op == RRC and pushreduce:
                pass                                   # staged push-reduce (R31)
            elif t.op == RRC:
                s.direct = s.pull = rv.direct = rv.pull = True
                s.kind, rv.kind = "psend", "prrc"
                rv.rem_buf = s.src_buf
            else:
                s.direct = rv.direct = True
                s.kind, rv.kind = "dsend", "drecv"
                s.rem_out = rv.dst_buf
                rv.store = False
        rv.pid = len(prims[t.dst]); prims[t.dst].append(rv); recv_of[i] = (t.dst, rv.pid)

    # -- connection activity + state-based merging (Eq. 7)
    act: Dict[int, Dict[Tuple[int, str], set]] = {r: {} for r in range(N)}
    for i, t in enumerate(tasks):
        act[t.src].setdefault((t.dst, "send"), set()).add(pidx[i])
        act[t.dst].setdefault((t.src, "recv"), set()).add(pidx[i])
    send_groups, recv_groups, lane_of_conn = {}, {}, {}
    for r in range(N):
        sa = {cn: a for cn, a in act[r].items() if cn[1] == "send"}
        ra = {cn: a for cn, a in act[r].items() if cn[1] == "recv"}
        send_groups[r] = _greedy_merge(sa)
        recv_groups[r] = _greedy_merge(ra)
        for gi, g in enumerate(send_groups[r]):
            for cn in g:
                lane_of_conn[(r, cn)] = gi
        for gi, g in enumerate(recv_groups[r]):
            for cn in g:
                lane_of_conn[(r, cn)] = gi
    for i, t in enumerate(tasks):
        r, p = send_of[i]
        prims[r][p].cta = lane_of_conn[(r, (t.dst, "send"))]; prims[r][p].lane = "S"
        r, p = recv_of[i]
        prims[r][p].cta = lane_of_conn[(r, (t.src, "recv"))]; prims[r][p].lane = "R"

    # -- local dependencies from the DAG
    def prim_at(i, x):
        t = tasks[i]
        return send_of[i][1] if t.src == x else recv_of[i][1]

    deps: Dict[int, Dict[int, set]] = {r: {p: set() for p in range(len(prims[r]))} for r in range(N)}
    for (u, v), ranks in edge_rank.items():
        for x in ranks:
            deps[x][prim_at(v, x)].add(prim_at(u, x))

    # -- fusion (recv-lane prim absorbs a same-CTA send whose only dependency it is)
    def fuse_plan():
        absorbed = {r: {} for r in range(N)}      # send pid -> fused recv pid
        for r in range(N):
            ps = prims[r]
            recv_lane = sorted((p for p in ps if p.lane == "R"), key=lambda p: (p.cta, p.pc))
            taken = set()
            for a in recv_lane:
                cands = [b for b in ps if b.lane == "S" and b.cta == a.cta and b.direct == a.direct
                         and b.pid not in taken and deps[r][b.pid] == {a.pid}]
                if not cands:
                    continue
                b = min(cands, key=lambda b: (b.pc, tasks[b.send_task].dst))
                taken.add(b.pid)
                absorbed[r][b.pid] = a.pid
        return absorbed

    absorbed = fuse_plan() if fuse else {r: {} for r in range(N)}

    def build(absorbed):
        out_prims: Dict[int, List[Prim]] = {}
        lanes: Dict[int, List[Tuple[List[int], List[int]]]] = {}
        for r in range(N):
            ps = [Prim(**{k: getattr(p, k) for k in p.__dataclass_fields__}) for p in prims[r]]
            for p in ps:
                p.deps = []
            fused_into = absorbed[r]
            for bpid, apid in fused_into.items():
                a, b = ps[apid], ps[bpid]
                t1 = a.recv_task
                t2 = b.send_task
                loc = (r, a.chunk)
                # readers of the value t1 writes, up to the next write of <r,c>
                acc = loc_acc[loc]
                pos = next(k for k, (_, i, _) in enumerate(acc) if i == t1 and acc[k][2] != "R")
                readers, final = set(), True
                for (_, i, kind) in acc[pos + 1:]:
                    if kind == "R":
                        readers.add(i)
                    else:
                        if kind == "RW":
                            readers.add(i)
                        final = False
                        break
                store = (final and is_output(coll, r, a.chunk)) or readers != {t2}
                a.send_task = t2
                if a.direct:     # value stays in our location; the send part keeps its mode
                    a.kind = DIRECT_FUSED[(a.kind, b.kind)]
                    a.rem_out = b.rem_out
                    if a.kind.startswith("drecv"):
                        a.src_buf = a.dst_buf
                    continue
                a.store = store
                a.kind = FUSED_KIND[(tasks[t1].op, store)]
                if not store:
                    a.dst_buf = None
            remap = {p.pid: fused_into.get(p.pid, p.pid) for p in ps}
            keep = [p for p in ps if p.pid not in fused_into]
            # copies for output locations never written on r
            copies = []
            written = {c for (rr, c) in first_w if rr == r}
            for c in range(ir.nchunks):
                if is_output(coll, r, c) and c not in written:
                    # the first data-moving send of the location from the send buffer also
                    # stores it locally; else a separate copy primitive (module docstring)
                    first = next((p for p in keep if p.chunk == c and p.kind in ("send", "dsend")
                                  and p.src_buf == "send"), None)
                    if first is not None:
                        first.store = True
                        first.dst_buf = "recv"
                        continue
                    cp = Prim(r, "copy", c, -1, src_buf="send", dst_buf="recv", cta=0, lane="R")
                    copies.append(cp)
            final_list = copies + keep
            newid = {}
            for k, p in enumerate(final_list):
                if p.pid >= 0 and p.kind != "copy":
                    newid[p.pid] = k
            raw_kind = {q.pid: q.kind for q in ps}

            def is_ack(d):   # dependency on a pull-send: completes with the peer's ack
                return direct and raw_kind[d] == "psend"

            for k, p in enumerate(final_list):
                old = p.pid
                p.pid = k
                if p.kind == "copy":
                    continue
                ds, acks = set(), set()
                srcs = list(deps[r][old])
                if old in fused_into.values():
                    for bpid, apid in fused_into.items():
                        if apid == old:
                            srcs += list(deps[r][bpid])
                for d in srcs:
                    (acks if is_ack(d) else ds).add(newid[remap[d]])
                ds.discard(k)
                acks.discard(k)
                p.deps = sorted(ds)
                p.ack_deps = sorted(acks)
            ncta = max(len(send_groups[r]), len(recv_groups[r]), 1)
            lane_lists = []
            for c in range(ncta):
                s_l = sorted((p for p in final_list if p.lane == "S" and p.cta == c),
                             key=lambda p: p.pc)
                r_l = sorted((p for p in final_list if p.lane == "R" and p.cta == c),
                             key=lambda p: p.pc)
                lane_lists.append(([p.pid for p in s_l], [p.pid for p in r_l]))
            # (ack dependencies are never implied by lane order)
            # drop dependencies implied by lane order
            pos_in_lane = {}
            for c, (sl, rl) in enumerate(lane_lists):
                for k, pid in enumerate(sl):
                    pos_in_lane[pid] = (c, "S", k)
                for k, pid in enumerate(rl):
                    pos_in_lane[pid] = (c, "R", k)
            for p in final_list:
                me = pos_in_lane[p.pid]
                p.deps = [d for d in p.deps
                          if not (pos_in_lane[d][:2] == me[:2] and pos_in_lane[d][2] < me[2])]
            for p in final_list:
                for d in p.deps:
                    final_list[d].has_counter = True
            out_prims[r] = final_list
            lanes[r] = lane_lists
        return out_prims, lanes

    out_prims, lanes = build(absorbed)
    any_fused = bool(fuse) and any(absorbed[r] for r in range(N))
    plan = Plan(ir, model, edges, edge_rank, Pr, pidx, out_prims, lanes,
                send_groups, recv_groups,
                {r: len(act[r]) for r in range(N)}, any_fused, direct)
    plan.pushreduce = bool(direct and pushreduce)
    plan._act = act
    if fuse and any(absorbed[r] for r in range(N)):
        from .replay import deadlock_free

        def rebuilt(ab, fused):
            op, ln = build(ab)
            pl = Plan(ir, model, edges, edge_rank, Pr, pidx, op, ln, send_groups, recv_groups,
                      {r: len(act[r]) for r in range(N)}, fused, direct)
            pl.pushreduce = bool(direct and pushreduce)
            pl._act = act
            return pl

        if not deadlock_free(plan, Ks=(1,), n_mbs=(1, 2, 3, 16)):
            # direct: fusions whose send part only posts "readable" add no wait edge
            safe = {r: {b: a for b, a in absorbed[r].items() if prims[r][b].kind == "psend"}
                    for r in range(N)} if direct else {r: {} for r in range(N)}
            plan = None
            if any(safe[r] for r in range(N)):
                plan = rebuilt(safe, True)
                if not deadlock_free(plan, Ks=(1,), n_mbs=(1, 2, 3, 16)):
                    plan = None
            if plan is None:
                plan = rebuilt({r: {} for r in range(N)}, False)
    return plan


def conn_positions(plan: Plan) -> Dict[Tuple[int, int], List[int]]:
    """FIFO order of every link (src, dst): its tasks sorted by pipeline index.
    The receiver consumes in this order (one recv lane per connection)."""
    pos: Dict[Tuple[int, int], List[int]] = {}
    for i, t in enumerate(plan.ir.transfers):
        pos.setdefault((t.src, t.dst), []).append(i)
    for k in pos:
        pos[k].sort(key=lambda i: plan.pidx[i])
    return pos
