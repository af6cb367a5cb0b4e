"""Oracle: wall-clock timeline of a plan under the paper's cost model.
TEST INFRASTRUCTURE ONLY.

Follows, in this order:

* Eq. 5: task-level execution.  Each lane runs its primitive list
  in order and every primitive runs all of its n micro-batch invocations.  An
  invocation starts as soon as the blocking model of the plan check allows it
  (``replay._Sim.enabled``: local dependencies, payload, FIFO credit and the direct
  transport's writable / readable flags).  Its effects apply when it ends
  (``replay._Sim.fire``).
* Cost of one invocation (reading R27): ``alpha + c * beta`` when it moves its
  c bytes over a link, else ``alpha``.  A link is moved over by a staged or pushed
  send, or by a pulled receive.  A FIFO drain, a flag post or a local copy moves
  nothing.  A push receiver's "writable" post takes no time.
* Eq. 1, T_conflict = n * z * (alpha + c * beta) + L(z) * gamma:
  - the z invocations moving data on one link share it, each at rate 1/z;
  - one that starts on a link already carrying others first waits
    gamma * L(z) / n, with L(z) = z - 1;
  - so z identical tasks of n invocations end at n * z * (alpha + c * beta) + L(z) * gamma.
  - The link is the (src, dst) connection under the pair model.  Under the port
    model it is both the sender's egress port and the receiver's ingress port, and
    the slower of the two sets the rate.
* Eq. 7 on the wall clock:
  - active_l(t) of a connection is the union of its invocations' [start, end)
    intervals;
  - connections of one direction whose activity never overlaps are merged
    greedily, in order of (first start, peer);
  - the result is the number of lanes the wall-clock state-based allocation needs.
"""
from __future__ import annotations

import math
from typing import Dict, List, Tuple

from .lower import PULL_SENDS, PUSH_RECVS, Plan
from .replay import Deadlock, _Sim


def _moves(p) -> List[Tuple]:
    """(link endpoints) this primitive moves bytes over: list of (src, dst)."""
    out = []
    if p.send_task is not None and not (p.direct and p.kind in PULL_SENDS):
        out.append(p.send_task)
    if p.direct and p.recv_task is not None and p.kind not in PUSH_RECVS:
        out.append(p.recv_task)
    return out


def timeline(plan: Plan, n_mb: int, K: int, instances: int, c: float, alpha: float, beta: float,
             gamma: float) -> Dict:
    sim = _Sim(plan, n_mb, instances, K)
    tasks = plan.ir.transfers

    def resources(p):
        res = []
        for t in _moves(p):
            x = tasks[t]
            if plan.model == "pair":
                res.append(("P", x.src, x.dst))
            else:
                res.append(("E", x.src))
                res.append(("I", x.dst))
        return res

    procs = sim.procs
    busy = [False] * len(procs)
    pen = [0.0] * len(procs)
    work = [0.0] * len(procs)
    start = [0.0] * len(procs)
    res = [[] for _ in procs]
    lane_busy = [0.0] * len(procs)
    load: Dict[Tuple, int] = {}
    active: Dict[Tuple[int, int, str], List[Tuple[float, float]]] = {}
    t = 0.0
    max_z = 1

    def z_of(i):
        return max([1] + [load.get(x, 0) for x in res[i]])

    while True:
        changed = True
        while changed:                                    # "writable" posts: no time
            changed = False
            for i, pr in enumerate(procs):
                if busy[i] or not sim.enabled(pr):
                    continue
                r, _, _, _, prog, k, _, phase = pr
                if plan.prims[r][prog[k]].kind in PUSH_RECVS and phase == 0:
                    sim.fire(pr)
                    changed = True
        starters = [i for i, pr in enumerate(procs) if not busy[i] and sim.enabled(pr)]
        starting: Dict[Tuple, int] = {}
        for i in starters:
            r, _, _, _, prog, k, _, _ = procs[i]
            res[i] = resources(plan.prims[r][prog[k]])
            for x in res[i]:
                starting[x] = starting.get(x, 0) + 1
        for i in starters:                                # simultaneous starters see the same z
            busy[i] = True
            start[i] = t
            work[i] = alpha + (c * beta if res[i] else 0.0)
            z0 = max([1] + [load.get(x, 0) + starting[x] for x in res[i]])
            pen[i] = gamma * (z0 - 1) / n_mb
        for i in starters:
            if pen[i] <= 0:
                for x in res[i]:
                    load[x] = load.get(x, 0) + 1
        if sim.finished():
            break
        if not any(busy):
            raise Deadlock("timeline: the plan deadlocks")
        zs = [z_of(i) if busy[i] and pen[i] <= 0 else 1 for i in range(len(procs))]
        max_z = max([max_z] + [zs[i] for i in range(len(procs)) if busy[i] and pen[i] <= 0])
        dt = math.inf
        for i in range(len(procs)):
            if busy[i]:
                dt = min(dt, pen[i] if pen[i] > 0 else work[i] * zs[i])
        t += dt
        eps = 1e-15 * max(1.0, t)
        for i in range(len(procs)):
            if not busy[i]:
                continue
            if pen[i] > 0:
                pen[i] -= dt
                if pen[i] <= eps:
                    pen[i] = 0.0
                    for x in res[i]:
                        load[x] = load.get(x, 0) + 1
                continue
            work[i] -= dt / zs[i]
        for i, pr in enumerate(procs):
            if not busy[i] or pen[i] > 0 or work[i] > eps:
                continue
            r, _, _, inst, prog, k, _, _ = pr
            p = plan.prims[r][prog[k]]
            for x in res[i]:
                load[x] -= 1
            busy[i] = False
            lane_busy[i] += t - start[i]
            if inst == 0:
                if p.send_task is not None:
                    active.setdefault((r, tasks[p.send_task].dst, "send"), []).append((start[i], t))
                if p.recv_task is not None:
                    active.setdefault((r, tasks[p.recv_task].src, "recv"), []).append((start[i], t))
            sim.fire(pr)

    merged = {}
    for r in range(plan.ir.nranks):
        for d in ("send", "recv"):
            conns = sorted((min(a for a, _ in iv), peer) for (rr, peer, dd), iv in active.items() if rr == r and dd == d)
            groups: List[List[Tuple[float, float]]] = []
            for _, peer in conns:
                iv = active[(r, peer, d)]
                for g in groups:
                    if not any(a0 < b1 and b0 < a1 for a0, a1 in iv for b0, b1 in g):
                        g.extend(iv)
                        break
                else:
                    groups.append(list(iv))
            merged[(r, d)] = len(groups)
    n = len(procs)
    comm = sum(lane_busy) / (n * t) if n and t > 0 else 0.0
    return {"makespan_s": t, "comm_time": comm, "avg_idle": 1.0 - comm if n else 0.0,
            "max_idle": max(1.0 - b / t for b in lane_busy) if n and t > 0 else 0.0, "max_z": max_z,
            "merged": merged, "active": active}
