"""Oracle: Alg. 1 HPDS and the round-robin baseline.  TEST INFRASTRUCTURE ONLY.

Alg. 1, explained in P:L1680-1774, transcribed line by line with
readings R2-R4:

* R2 link model.  ``pair``: a task's link is its (src, dst) connection.  ``port``:
  a task occupies egress(src) and ingress(dst); two tasks conflict when they
  share either port.
* R3 priority.  Every chunk starts at 0 and loses 1 each time its NodeList is
  inserted (line 20); "lower execution frequency => higher priority"
  (P:L1748-1758).  GetHighestWithFlag takes the highest priority among chunks whose
  flag is true; ties go to the lowest ChunkId.
* R4 readiness / comm check.  "without data dependency" (line 11) = every DAG
  predecessor already removed from G (line 22), evaluated when the inner
  iteration starts.  Line 12 checks the task's link against Pc and the NodeList
  built so far.  Candidates are visited in (step, src, dst) order.
"""
from __future__ import annotations

from typing import List, Sequence

from .dag import preds_succs


def links(t, model: str):
    if model == "pair":
        return {("pair", t.src, t.dst)}
    if model == "port":
        return {("out", t.src), ("in", t.dst)}
    raise ValueError(model)


def hpds(ir, edges, model: str = "pair") -> List[List[int]]:
    """Return Pr = [Pc0, Pc1, ...], each Pc a list of task indices in insertion order."""
    tasks = ir.transfers
    n = len(tasks)
    preds, _ = preds_succs(n, edges)
    chunks = sorted({t.chunk for t in tasks})
    G = set(range(n))                                   # line 1 input
    prio = {c: 0 for c in chunks}                       # line 3 Q
    Pr: List[List[int]] = []                            # line 4
    while G:                                            # line 5
        Pc: List[int] = []                              # line 6
        used = set()
        F = {c: True for c in chunks}                   # line 7
        while any(F.values()):                          # line 8
            C = max((c for c in chunks if F[c]), key=lambda c: (prio[c], -c))  # line 9
            node_list: List[int] = []                   # line 10
            ready = [i for i in G if tasks[i].chunk == C and not (preds[i] & G)]
            ready.sort(key=lambda i: (tasks[i].step, tasks[i].src, tasks[i].dst))
            for i in ready:                             # line 11
                li = links(tasks[i], model)
                if not (li & used):                     # line 12
                    node_list.append(i)                 # line 13
                    used |= li
            if not node_list:                           # line 16
                F[C] = False                            # line 17
            else:
                Pc.extend(node_list)                    # line 19
                prio[C] -= 1                            # line 20-21
                G -= set(node_list)                     # line 22
        if not Pc:
            raise RuntimeError("HPDS made no progress (cyclic dependencies?)")
        Pr.append(Pc)                                   # line 25
    return Pr


def round_robin(ir, edges, model: str = "pair") -> List[List[int]]:
    """RR baseline: chunks visited in ascending ChunkId order in a
    circular queue with an immutable sequence (no priorities).  A sub-pipeline is
    built by repeated passes over chunks 0..C-1 until a whole pass adds nothing."""
    tasks = ir.transfers
    n = len(tasks)
    preds, _ = preds_succs(n, edges)
    chunks = sorted({t.chunk for t in tasks})
    G = set(range(n))
    Pr = []
    while G:
        Pc: List[int] = []
        used = set()
        progress = True
        while progress:
            progress = False
            for C in chunks:
                ready = [i for i in G if tasks[i].chunk == C and not (preds[i] & G)]
                ready.sort(key=lambda i: (tasks[i].step, tasks[i].src, tasks[i].dst))
                nl = []
                for i in ready:
                    li = links(tasks[i], model)
                    if not (li & used):
                        nl.append(i)
                        used |= li
                if nl:
                    Pc.extend(nl)
                    G -= set(nl)
                    progress = True
        if not Pc:
            raise RuntimeError("RR made no progress")
        Pr.append(Pc)
    return Pr


def pipeline_index(Pr: Sequence[Sequence[int]], ntasks: int) -> List[int]:
    pidx = [-1] * ntasks
    for k, pc in enumerate(Pr):
        for i in pc:
            pidx[i] = k
    return pidx
