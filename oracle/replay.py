"""Oracle: schedule replay and invariants I1-I6.
TEST INFRASTRUCTURE ONLY.

The fp result of a schedule depends on its association order, so besides the
definition (definition.py) the oracle replays the plan itself on host buffers:

1. ``symbolic``: every location holds the set of ranks whose inputs it contains;
   recv copies the set, rrc unions two disjoint sets (I1); at the end every rank
   holds the full result (I3).  Tasks are applied in step order (reading R1).
2. ``replay``: a blocking simulator executes the lowered plan at (primitive,
   micro-batch, instance) granularity.  Every lane of every CTA of every rank and
   instance is a sequential process running its pipeline-ordered primitive list,
   each primitive looping over all micro-batches (task-level execution).
   Wait rules (staged FIFO mode, reading R5):
     - a primitive waits, for micro-batch j, until each of its local dependencies
       has finished micro-batch j (rule (1));
     - consuming a payload waits until the sender has put it in the FIFO of that
       link (one FIFO per link and instance, depth K, filled in pipeline order);
     - producing a payload waits for FIFO credit (fewer than K unconsumed slots).
   Values: send FIFO <- local; recv local <- FIFO; rrc local <- local (+) FIFO;
   rrs next FIFO <- local (+) FIFO; rcs local, next FIFO <- FIFO (numerics.combine).
3. ``happens_before_races``: vector clocks over the same execution prove that
   every pair of conflicting accesses (buffer slices and FIFO slots, >= 1 write)
   is ordered by program order, FIFO and counter synchronisation (I2).
4. ``deadlock_free``: the control-only simulation completes (I4).

Geometry (reading R6): AllReduce chunk c covers elements
[c*C, (c+1)*C) with C = ceil(count / N) rounded up to 256 bytes; AllGather /
ReduceScatter chunk c is rank c's segment.  Micro-batch j of a chunk is its
j-th M-element slice, M = min(chunkBytes/elt, C rounded up to 16 B); each
micro-batch is split into ``instances`` contiguous 16-byte-aligned slices.
"""
from __future__ import annotations

import random
from collections import defaultdict
from typing import Dict, List, Optional, Tuple

import numpy as np

from .lower import PULL_SENDS, PUSH_RECVS, Plan, conn_positions, is_output
from .numerics import combine

ELT = {"int32": 4, "float32": 4, "float16": 2, "bfloat16": 2}
STORE = {"int32": np.int32, "float32": np.float32, "float16": np.float16, "bfloat16": np.uint16}
POISON = {"int32": 0x5A5A5A5A, "float32": 0x7FC5A5A5, "float16": 0x7E55, "bfloat16": 0x7FC5}


def _cdiv(a, b):
    return -(-a // b)


def _rup(a, b):
    return _cdiv(a, b) * b


class Geometry:
    def __init__(self, coll: str, nranks: int, count: int, elt: int,
                 chunk_bytes: int, instances: int):
        self.coll, self.nranks, self.count, self.elt = coll, nranks, count, elt
        vec = 16 // elt
        if coll == "allreduce":
            C = _rup(_cdiv(count, nranks), 256 // elt) if count else 0
            self.chunk_len = [max(0, min(C, count - c * C)) for c in range(nranks)]
        else:
            C = count
            self.chunk_len = [count] * nranks
        self.C = C
        M = max(chunk_bytes // elt, vec)
        self.M = min(M, _rup(C, vec)) if C else M
        self.n_mb = _cdiv(C, self.M) if C else 0
        self.Mi = _rup(_cdiv(self.M, instances), vec)
        self.instances = instances

    def slice(self, c: int, j: int, i: int) -> Tuple[int, int]:
        lo = j * self.M + i * self.Mi
        hi = min(lo + self.Mi, (j + 1) * self.M, self.chunk_len[c])
        lo = min(lo, hi)
        return lo, hi

    def chunk_off(self, buf: str, c: int) -> int:
        if self.coll == "allreduce":
            return c * self.C
        if self.coll == "allgather":
            return 0 if buf == "send" else c * self.C
        return 0 if buf == "recv" else c * self.C           # reducescatter


# ------------------------------------------------------------------ symbolic pass

def symbolic(ir) -> Dict[Tuple[int, int], Optional[frozenset]]:
    """I1 (exactly-once / disjoint unions) and the final contents for I3."""
    N = ir.nranks
    loc = {}
    for r in range(N):
        for c in range(ir.nchunks):
            if ir.coll == "allgather":
                loc[(r, c)] = frozenset([r]) if r == c else None
            else:
                loc[(r, c)] = frozenset([r])
    for t in sorted(ir.transfers, key=lambda t: t.step):
        s = loc[(t.src, t.chunk)]
        if s is None:
            raise AssertionError(f"I6: read of undefined location by {t}")
        d = loc[(t.dst, t.chunk)]
        if t.op == "recv":
            if ir.coll == "allgather" and d is not None:
                raise AssertionError(f"I1: location written twice by {t}")
            loc[(t.dst, t.chunk)] = s
        else:
            if d & s:
                raise AssertionError(f"I1: overlapping contributions {sorted(d & s)} in {t}")
            loc[(t.dst, t.chunk)] = d | s
    return loc


def check_full_result(ir, loc) -> None:
    """I3: AR every <r,c> = all ranks; AG <r,c> = {c}; RS <r,r> = all ranks."""
    full = frozenset(range(ir.nranks))
    for r in range(ir.nranks):
        for c in range(ir.nchunks):
            v = loc[(r, c)]
            if ir.coll == "allreduce" and v != full:
                raise AssertionError(f"I3: AR <{r},{c}> holds {v}")
            if ir.coll == "allgather" and v != frozenset([c]):
                raise AssertionError(f"I3: AG <{r},{c}> holds {v}")
            if ir.coll == "reducescatter" and c == r and v != full:
                raise AssertionError(f"I3: RS <{r},{r}> holds {v}")


# ------------------------------------------------------------------ simulator

class Deadlock(RuntimeError):
    pass


class _Sim:
    """Processes = lanes x instances.  Per (link, instance): posted payload positions
    (``fifo``) and a monotone ``credit``: the receiver's consumption (staged), its
    "writable" posts (direct push) or its read acknowledgements (direct pull)."""

    def __init__(self, plan: Plan, n_mb: int, instances: int, K: int, rings: Optional[str] = None):
        self.plan, self.n_mb, self.I, self.K = plan, n_mb, instances, K
        # Device-faithful flag model (R26): each payload flag lives in slot pos % K of a
        # ring, overwritten with pos + 1 on every post; the receiver of pos tests
        # "slot >= pos + 1".  rings="link": one ring per (link, instance); rings="lane":
        # one ring per (link, instance, sending lane).  Every test of the device
        # condition that disagrees with the ideal "pos was posted and not consumed"
        # is recorded in self.hazards.
        self.rings = rings
        self.slots = defaultdict(dict)
        self.hazards = []
        self.send_lane = {}
        for r, prims in plan.prims.items():
            for pid, p in enumerate(prims):
                if p.send_task is not None:
                    self.send_lane[p.send_task] = (p.cta, p.lane)
        self.tasks = plan.ir.transfers
        order = conn_positions(plan)
        self.tpos = {}
        for link, lst in order.items():
            for k, i in enumerate(lst):
                self.tpos[i] = k
        self.procs = []
        for r, ctas in plan.lanes.items():
            for c, (sl, rl) in enumerate(ctas):
                for lane, prog in (("S", sl), ("R", rl)):
                    if prog:
                        for inst in range(instances):
                            self.procs.append([r, c, lane, inst, prog, 0, 0, 0])   # ..., k, j, phase
        self.done = defaultdict(int)
        self.fifo = defaultdict(dict)        # (link, inst) -> {pos: payload}
        self.credit = defaultdict(int)
        self.events = 0

    def _link(self, i):
        t = self.tasks[i]
        return (t.src, t.dst)

    def pos(self, task, j):
        return self.tpos[task] * self.n_mb + j

    def deps_ok(self, r, p, j, inst) -> bool:
        for d in p.deps:
            if self.done[(r, d, inst)] < j + 1:
                return False
        for d in p.ack_deps:
            t = self.plan.prims[r][d].send_task
            if self.credit[(self._link(t), inst)] < self.pos(t, j) + 1:
                return False
        return True

    def send_ok(self, p, j, inst) -> bool:
        if p.send_task is None:
            return True
        pos = self.pos(p.send_task, j)
        cr = self.credit[(self._link(p.send_task), inst)]
        if not p.direct:
            return pos < cr + self.K
        if p.kind in PULL_SENDS:                      # pull-send: post "readable"
            return True
        return cr >= pos + 1                          # push: receiver location writable

    def _ring(self, task, inst):
        key = (self._link(task), inst)
        return key + (self.send_lane[task],) if self.rings == "lane" else key

    def _arrived(self, task, j, inst) -> bool:
        pos = self.pos(task, j)
        ideal = pos in self.fifo[(self._link(task), inst)]
        if self.rings:
            dev = self.slots[self._ring(task, inst)].get(pos % self.K, 0) >= pos + 1
            if dev != ideal:
                self.hazards.append((self._link(task), inst, pos, "early" if dev else "lost"))
        return ideal

    def enabled(self, pr) -> bool:
        r, c, lane, inst, prog, k, j, phase = pr
        if k >= len(prog):
            return False
        p = self.plan.prims[r][prog[k]]
        if p.kind == "copy":
            return True
        if p.kind in PUSH_RECVS and phase == 1:       # push receiver waiting for the payload
            return self._arrived(p.recv_task, j, inst) and self.send_ok(p, j, inst)
        if not self.deps_ok(r, p, j, inst):
            return False
        if p.kind in PUSH_RECVS:                      # phase 0: post "writable"
            return True
        if p.recv_task is not None:
            if not self._arrived(p.recv_task, j, inst):
                return False
        return self.send_ok(p, j, inst)

    def finished(self) -> bool:
        return all(pr[5] >= len(pr[4]) for pr in self.procs)

    def fire(self, pr, action=None):
        r, c, lane, inst, prog, k, j, phase = pr
        p = self.plan.prims[r][prog[k]]
        if p.kind in PUSH_RECVS and phase == 0:       # post "writable", keep the micro-batch
            key = (self._link(p.recv_task), inst)
            self.credit[key] = max(self.credit[key], self.pos(p.recv_task, j) + 1)
            pr[7] = 1
            self.events += 1
            return
        pr[7] = 0
        incoming = None
        if p.recv_task is not None:
            key = (self._link(p.recv_task), inst)
            pos = self.pos(p.recv_task, j)
            incoming = self.fifo[key].pop(pos)
            if not p.direct:
                assert pos == self.credit[key], "out-of-order consumption"
                self.credit[key] += 1
            elif p.kind not in PUSH_RECVS:            # pull: read acknowledged
                self.credit[key] = max(self.credit[key], pos + 1)
        out = action(p, r, j, inst, incoming) if action else None
        if p.send_task is not None:
            key = (self._link(p.send_task), inst)
            self.fifo[key][self.pos(p.send_task, j)] = out
            if self.rings:
                pos = self.pos(p.send_task, j)
                self.slots[self._ring(p.send_task, inst)][pos % self.K] = pos + 1
        if p.kind != "copy":
            self.done[(r, prog[k], inst)] = j + 1
        j += 1
        if j >= (self.n_mb if p.kind != "copy" else 1):
            k, j = k + 1, 0
        pr[5], pr[6] = k, j
        self.events += 1

    def run(self, sched: str = "rr", seed: int = 0, action=None, on_fire=None):
        rng = random.Random(seed)
        n = len(self.procs)
        if sched == "rr":
            idle = 0
            idx = 0
            while not self.finished():
                pr = self.procs[idx]
                if self.enabled(pr):
                    if on_fire:
                        on_fire(pr, "pre")
                    self.fire(pr, action)
                    idle = 0
                else:
                    idle += 1
                    if idle > n:
                        raise Deadlock(self._stuck())
                idx = (idx + 1) % n
        else:
            while not self.finished():
                en = [pr for pr in self.procs if self.enabled(pr)]
                if not en:
                    raise Deadlock(self._stuck())
                pr = rng.choice(en)
                if on_fire:
                    on_fire(pr, "pre")
                self.fire(pr, action)

    def _stuck(self):
        out = []
        for r, c, lane, inst, prog, k, j, _ in self.procs:
            if k < len(prog):
                p = self.plan.prims[r][prog[k]]
                out.append(f"rank{r} cta{c} {lane} inst{inst} at {p.kind} chunk{p.chunk} mb{j}")
        return "deadlock: " + "; ".join(out[:12])


def deadlock_free(plan: Plan, Ks=(1, 2, 8), n_mbs=(1, 2, 16), instances=(1,)) -> bool:
    """I4: the control-only simulation completes for every (K, n_mb, instances)."""
    for K in Ks:
        for n_mb in n_mbs:
            for I in instances:
                try:
                    _Sim(plan, n_mb, I, K).run("rr")
                except Deadlock:
                    return False
    return True


# ------------------------------------------------------------------ value replay

def make_buffers(plan: Plan, inputs: List[np.ndarray], dtype: str, count: int,
                 inplace: bool = False):
    ir = plan.ir
    N = ir.nranks
    st = STORE[dtype]
    bufs = []
    for r in range(N):
        x = np.asarray(inputs[r]).astype(st, copy=True)
        if ir.coll == "allreduce":
            if inplace:
                b = {"send": x, "recv": x}
            else:
                rv = np.empty(count, dtype=st)
                rv.view(np.uint16 if st in (np.float16, np.uint16) else np.uint32)[:] = POISON[dtype]
                b = {"send": x, "recv": rv}
        elif ir.coll == "allgather":
            rv = np.empty(N * count, dtype=st)
            rv.view(np.uint16 if st in (np.float16, np.uint16) else np.uint32)[:] = POISON[dtype]
            if inplace:
                rv[r * count:(r + 1) * count] = x
                b = {"send": rv[r * count:(r + 1) * count], "recv": rv}
            else:
                b = {"send": x, "recv": rv}
        else:
            sc = np.empty(N * count, dtype=st)
            if inplace:
                b = {"send": x, "recv": x[r * count:(r + 1) * count], "scratch": sc}
            else:
                rv = np.empty(count, dtype=st)
                rv.view(np.uint16 if st in (np.float16, np.uint16) else np.uint32)[:] = POISON[dtype]
                b = {"send": x, "recv": rv, "scratch": sc}
        bufs.append(b)
    return bufs


def replay(plan: Plan, inputs: List[np.ndarray], dtype: str, count: int, op: str = "sum",
           chunk_bytes: int = 1 << 20, instances: int = 1, K: int = 4,
           sched: str = "rr", seed: int = 0, inplace: bool = False):
    """Execute the plan on host buffers; returns each rank's receive buffer."""
    ir = plan.ir
    g = Geometry(ir.coll, ir.nranks, count, ELT[dtype], chunk_bytes, instances)
    bufs = make_buffers(plan, inputs, dtype, count, inplace)
    if count == 0 or g.n_mb == 0:
        return [b["recv"] for b in bufs]
    sim = _Sim(plan, g.n_mb, instances, K)

    def action(p, r, j, inst, incoming):
        if p.kind == "copy":                          # local copy of an unwritten output
            so, do = g.chunk_off("send", p.chunk), g.chunk_off("recv", p.chunk)
            for jx in range(g.n_mb):
                lo, hi = g.slice(p.chunk, jx, inst)
                bufs[r]["recv"][do + lo:do + hi] = bufs[r]["send"][so + lo:so + hi]
            return None
        lo, hi = g.slice(p.chunk, j, inst)
        tasks = plan.ir.transfers
        if p.kind in ("dsend", "drecv_d"):            # direct push: write the receiver's location
            o = g.chunk_off(p.src_buf, p.chunk)
            d, od = tasks[p.send_task].dst, g.chunk_off(p.rem_out, p.chunk)
            bufs[d][p.rem_out][od + lo:od + hi] = bufs[r][p.src_buf][o + lo:o + hi]
            if p.kind == "dsend" and p.store:         # ... and the local copy of an unwritten output
                od2 = g.chunk_off(p.dst_buf, p.chunk)
                bufs[r][p.dst_buf][od2 + lo:od2 + hi] = bufs[r][p.src_buf][o + lo:o + hi]
            return None
        if p.kind in ("psend", "drecv", "drecv_p"):   # flags only
            return None
        if p.kind in ("prrc", "prrc_p", "prrc_d"):    # direct pull: read the sender's location
            s_, os_ = tasks[p.recv_task].src, g.chunk_off(p.rem_buf, p.chunk)
            incoming = bufs[s_][p.rem_buf][os_ + lo:os_ + hi].copy()
        if p.recv_task is None:                       # plain send
            o = g.chunk_off(p.src_buf, p.chunk)
            if p.store:                               # ... storing an unwritten output locally too
                od2 = g.chunk_off(p.dst_buf, p.chunk)
                bufs[r][p.dst_buf][od2 + lo:od2 + hi] = bufs[r][p.src_buf][o + lo:o + hi]
            return bufs[r][p.src_buf][o + lo:o + hi].copy()
        if p.reduce:
            o = g.chunk_off(p.src_buf, p.chunk)
            v = combine(bufs[r][p.src_buf][o + lo:o + hi], incoming, dtype, op)
        else:
            v = incoming
        if p.store:
            o = g.chunk_off(p.dst_buf, p.chunk)
            bufs[r][p.dst_buf][o + lo:o + hi] = v
        if p.kind == "prrc_d":                        # ... and push it to the next hop
            d, od = tasks[p.send_task].dst, g.chunk_off(p.rem_out, p.chunk)
            bufs[d][p.rem_out][od + lo:od + hi] = v
            return None
        if p.kind == "prrc_p":
            return None
        return v.copy() if p.send_task is not None else None

    sim.run(sched, seed, action)
    return [b["recv"] for b in bufs]


# ------------------------------------------------------------------ I2 happens-before

def happens_before_races(plan: Plan, n_mb: int = 2, instances: int = 1, K: int = 1, inplace: bool = False):
    """Return the list of conflicting, unordered access pairs (empty = I2 holds).

    Memory cells are (rank, buffer, chunk, micro-batch, instance) slices and FIFO
    slots (link, instance, pos mod K).  Synchronisation edges: program order; a
    payload/flag post of a position -> its consumer; a credit post of a position ->
    the waiter it enables (staged: the sender of position p+K; direct push: the
    sender of p; direct pull: dependents of the pull-send); a primitive's micro-batch j
    -> waits on its counter for j."""
    sim = _Sim(plan, n_mb, instances, K)
    P = len(sim.procs)
    pid_of = {id(pr): k for k, pr in enumerate(sim.procs)}
    vc = [[0] * P for _ in range(P)]
    put_vc, credit_vc, done_vc = {}, {}, {}
    cells = defaultdict(list)     # cell -> [(proc, own_clock, vc_snapshot, is_write)]
    tasks = plan.ir.transfers

    def on_fire(pr, _):
        me = pid_of[id(pr)]
        r, c, lane, inst, prog, k, j, phase = pr
        p = plan.prims[r][prog[k]]
        v = vc[me]

        def join(o):
            for q in range(P):
                if o[q] > v[q]:
                    v[q] = o[q]

        acc = []
        rlink = sim._link(p.recv_task) if p.recv_task is not None else None
        slink = sim._link(p.send_task) if p.send_task is not None else None
        rpos = sim.pos(p.recv_task, j) if p.recv_task is not None else None
        spos = sim.pos(p.send_task, j) if p.send_task is not None else None
        push_recv = p.kind in PUSH_RECVS

        def send_joins():
            if p.send_task is not None:
                if not p.direct:
                    if spos - K >= 0:
                        join(credit_vc[(slink, inst, spos - K)])
                elif p.kind not in PULL_SENDS:
                    join(credit_vc[(slink, inst, spos)])

        if push_recv and phase == 1:
            join(put_vc[(rlink, inst, rpos)])
            send_joins()
        elif p.kind != "copy":
            for d in p.deps:
                join(done_vc[(r, d, inst, j)])
            for d in p.ack_deps:
                t = plan.prims[r][d].send_task
                join(credit_vc[(sim._link(t), inst, sim.pos(t, j))])
            if not push_recv:
                if p.recv_task is not None:
                    join(put_vc[(rlink, inst, rpos)])
                send_joins()
        jj = 0 if p.kind == "copy" else j
        if p.kind == "copy":
            acc.append(((r, "send", p.chunk, -1, -1), False))
            acc.append(((r, "recv", p.chunk, -1, -1), True))
        elif p.kind in ("dsend", "drecv_d"):
            if not (push_recv and phase == 0):
                acc.append(((r, p.src_buf, p.chunk, jj, inst), False))
                acc.append(((tasks[p.send_task].dst, p.rem_out, p.chunk, jj, inst), True))
                if p.kind == "dsend" and p.store and not inplace:  # local copy of an unwritten output
                    acc.append(((r, p.dst_buf, p.chunk, jj, inst), True))
        elif p.kind in ("prrc", "prrc_p", "prrc_d"):
            acc.append(((tasks[p.recv_task].src, p.rem_buf, p.chunk, jj, inst), False))
            acc.append(((r, p.src_buf, p.chunk, jj, inst), False))
            acc.append(((r, p.dst_buf, p.chunk, jj, inst), True))
            if p.kind == "prrc_d":
                acc.append(((tasks[p.send_task].dst, p.rem_out, p.chunk, jj, inst), True))
        elif p.kind not in ("psend", "drecv", "drecv_p"):
            if p.recv_task is not None:
                acc.append((("fifo", rlink, inst, rpos % K), False))
            if p.send_task is not None:
                acc.append((("fifo", slink, inst, spos % K), True))
            if p.src_buf and (p.recv_task is None or p.reduce):
                acc.append(((r, p.src_buf, p.chunk, jj, inst), False))
            if p.recv_task is not None and p.store:
                acc.append(((r, p.dst_buf, p.chunk, jj, inst), True))
            if p.recv_task is None and p.store and not inplace:  # send storing an unwritten output
                acc.append(((r, p.dst_buf, p.chunk, jj, inst), True))
        if inplace and p.kind == "copy":
            acc = []  # in-place, the output already holds the input: the copy does nothing
        if inplace:  # in-place: a location's send- and receive-buffer copies are one memory
            acc = [((cl[0], "recv" if cl[1] == "send" else cl[1]) + cl[2:], w) if cl[0] != "fifo" else (cl, w)
                   for cl, w in acc]
        v[me] += 1
        snap = list(v)
        for cell, w in acc:
            if cell[0] == "fifo" or cell[3] >= 0:
                cells[cell].append((me, v[me], snap, w))
            else:  # copy touches every micro-batch/instance slice of the chunk
                for jx in range(n_mb):
                    for ix in range(instances):
                        cells[(cell[0], cell[1], cell[2], jx, ix)].append((me, v[me], snap, w))
        if push_recv and phase == 0:
            credit_vc[(rlink, inst, rpos)] = snap          # "writable"
            return
        if p.recv_task is not None and not push_recv:
            credit_vc[(rlink, inst, rpos)] = snap          # consumed / read acknowledged
        if p.send_task is not None:
            put_vc[(slink, inst, spos)] = snap             # payload / "written" / "readable"
        if p.kind != "copy":
            done_vc[(r, prog[k], inst, j)] = snap

    sim.run("rr", 0, None, on_fire)
    races = []
    for cell, acc in cells.items():
        for a in range(len(acc)):
            for b in range(a + 1, len(acc)):
                pa, ca, va, wa = acc[a]
                pb, cb, vb, wb = acc[b]
                if not (wa or wb) or pa == pb:
                    continue
                if not (vb[pa] >= ca or va[pb] >= cb):
                    races.append((cell, acc[a][:2], acc[b][:2]))
    # send-buffer reads of RS/AR aliasing: in-place runs map "send" and "recv" to one
    # array, so a read of <r,c> from "send" must precede every write of <r,c>.
    return races


# ------------------------------------------------------------------ I5

def check_plan(plan: Plan) -> None:
    ir = plan.ir
    tasks = ir.transfers
    seen = sorted(i for pc in plan.Pr for i in pc)
    assert seen == list(range(len(tasks))), "I5: each task in exactly one Pc"
    from .hpds import links
    for pc in plan.Pr:
        used = set()
        for i in pc:
            li = links(tasks[i], plan.model)
            assert not (li & used), "I5: two tasks of a Pc share a link"
            used |= li
    for u, v in plan.edges:
        assert plan.pidx[u] <= plan.pidx[v], "I5: predecessor in a later Pc"
    for r, ctas in plan.lanes.items():
        for sl, rl in ctas:
            for lane in (sl, rl):
                pcs = [plan.prims[r][p].pc for p in lane if plan.prims[r][p].kind != "copy"]
                assert len(pcs) == len(set(pcs)), "I5: two primitives of a lane share a Pc"
                assert pcs == sorted(pcs)
        for groups in (plan.send_groups[r], plan.recv_groups[r]):
            for g in groups:
                acc = set()
                for cn in g:
                    a = plan._act[r][cn]
                    assert not (acc & a), "I5: merged connections overlap in time"
                    acc |= a
        sb, rb = plan.clique_bound(r)
        assert len(plan.send_groups[r]) >= sb and len(plan.recv_groups[r]) >= rb


# ------------------------------------------------------------------ step-order dataflow (sampled)

def dataflow_values(ir, chunk_inputs, dtype: str, op: str = "sum"):
    """The IR executed literally in step order on per-chunk value vectors.

    ``chunk_inputs[r][c]`` is rank r's input restricted to any set of element
    positions of chunk c (the same positions for every rank); returns
    ``out[r][c]`` at those positions.  Because every element of a chunk follows
    the same transfers, this gives the schedule's exact result (same association
    order as ``replay``, R8) for sampled elements of arbitrarily large buffers.
    Locations never written keep their input (AG: owner's chunk only is defined)."""
    N = ir.nranks
    val = {}
    for r in range(N):
        for c in range(ir.nchunks):
            if ir.coll == "allgather":
                val[(r, c)] = chunk_inputs[r][c] if r == c else None
            else:
                val[(r, c)] = chunk_inputs[r][c]
    for t in sorted(ir.transfers, key=lambda t: t.step):
        incoming = val[(t.src, t.chunk)]
        if t.op == "recv":
            val[(t.dst, t.chunk)] = incoming.copy()
        else:
            val[(t.dst, t.chunk)] = combine(val[(t.dst, t.chunk)], incoming, dtype, op)
    return [[val[(r, c)] for c in range(ir.nchunks)] for r in range(N)]
