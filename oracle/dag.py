"""Oracle: global dependency analysis -> DAG G_A = (V_T, E).  TEST INFRASTRUCTURE ONLY.

Follows P:L705-714 (data dependency: two tasks access the same buffer offset),
P:L813-826 (edge v_i -> v_j: v_j consumes data produced by v_i), P:L1420-1440 and
P:L1657-1664 (same ChunkId: later Step depends on earlier; different ChunkIds
independent), under reading R1:

* A location is <rank, chunk>.  Task t = (s, d, step, c, op) reads <s,c>; an
  ``rrc`` also reads <d,c>; every task writes <d,c>.
* Per location, accesses are ordered by step.  A write depends on the last write
  (WAW) and on every read since it (WAR); a read depends on the last write (RAW).
* Two accesses to one location at the same step, at least one a write, make the
  IR invalid (R1/R9).  Edges never join different chunks.

Each edge records the rank of the location that induced it; the lowering turns
it into a local dependency on that rank.
"""
from __future__ import annotations

from collections import defaultdict
from typing import Dict, List, Set, Tuple

from .ir import IR, RRC, RECV


class InvalidIR(ValueError):
    pass


def accesses(t) -> List[Tuple[Tuple[int, int], str]]:
    """(location, kind) pairs of a transfer; kind in {"R", "W", "RW"}."""
    acc = [((t.src, t.chunk), "R")]
    acc.append(((t.dst, t.chunk), "RW" if t.op == RRC else "W"))
    return acc


def validate(ir: IR) -> None:
    """I6: ranks/chunks in range, no self transfer, op known, coll-specific rules."""
    if ir.coll not in ("allgather", "reducescatter", "allreduce"):
        raise InvalidIR(f"unknown coll {ir.coll}")
    if ir.nchunks != ir.nranks:
        raise InvalidIR("nchunks must equal nranks (R19)")
    for t in ir.transfers:
        if not (0 <= t.src < ir.nranks and 0 <= t.dst < ir.nranks):
            raise InvalidIR(f"rank out of range: {t}")
        if not 0 <= t.chunk < ir.nchunks:
            raise InvalidIR(f"chunk out of range: {t}")
        if t.src == t.dst:
            raise InvalidIR(f"self transfer: {t}")
        if t.op not in (RECV, RRC):
            raise InvalidIR(f"bad op: {t}")
        if t.step < 0:
            raise InvalidIR(f"negative step: {t}")
        if ir.coll == "allgather" and t.op == RRC:
            raise InvalidIR("allgather algorithms use recv only")
    if len(set(ir.transfers)) != len(ir.transfers):
        raise InvalidIR("duplicate transfer")


def build_dag(ir: IR):
    """Return (edges, edge_rank) where edges is a sorted list of (u, v) task-index
    pairs and edge_rank maps (u, v) -> set of ranks of the inducing locations."""
    validate(ir)
    by_loc: Dict[Tuple[int, int], List[Tuple[int, int, str]]] = defaultdict(list)
    for i, t in enumerate(ir.transfers):
        for loc, kind in accesses(t):
            by_loc[loc].append((t.step, i, kind))
    edge_rank: Dict[Tuple[int, int], Set[int]] = defaultdict(set)
    for loc, acc in by_loc.items():
        acc.sort()
        # same-step conflict check
        steps: Dict[int, List[Tuple[int, str]]] = defaultdict(list)
        for step, i, kind in acc:
            steps[step].append((i, kind))
        last_w = None
        readers: List[int] = []
        for step in sorted(steps):
            group = steps[step]
            has_write = any(k != "R" for _, k in group)
            if has_write and len(group) > 1:
                raise InvalidIR(f"same-step conflict at location {loc}, step {step}")
            if not has_write:
                for i, _ in group:
                    if last_w is not None:
                        edge_rank[(last_w, i)].add(loc[0])
                    readers.append(i)
            else:
                i, _ = group[0]
                if last_w is not None:
                    edge_rank[(last_w, i)].add(loc[0])
                for rd in readers:
                    if rd != i:
                        edge_rank[(rd, i)].add(loc[0])
                last_w = i
                readers = []
    edges = sorted(edge_rank)
    return edges, dict(edge_rank)


def preds_succs(ntasks: int, edges):
    preds = [set() for _ in range(ntasks)]
    succs = [set() for _ in range(ntasks)]
    for u, v in edges:
        preds[v].add(u)
        succs[u].add(v)
    return preds, succs


def check_defined_reads(ir: IR) -> None:
    """I6 (reads never touch undefined locations) + AG write-once rule.

    AllGather: initially only <r,r> is defined; every other location must be
    written exactly once, by a recv, before it is read.  RS/AR: every location is
    defined initially."""
    if ir.coll != "allgather":
        return
    first_write: Dict[Tuple[int, int], int] = {}
    for t in ir.transfers:
        loc = (t.dst, t.chunk)
        if loc[0] == loc[1]:
            raise InvalidIR(f"allgather overwrites the owner's chunk: {t}")
        if loc in first_write:
            raise InvalidIR(f"allgather location written twice: {loc}")
        first_write[loc] = t.step
    for t in ir.transfers:
        loc = (t.src, t.chunk)
        if loc[0] == loc[1]:
            continue
        if loc not in first_write or first_write[loc] >= t.step:
            raise InvalidIR(f"read of undefined location {loc} by {t}")
