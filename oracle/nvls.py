"""Oracle: the NVLS (NVLink SHARP) schedule of SURVEY §8(f) f3.  TEST INFRASTRUCTURE ONLY.

Not in the paper: f3 is the B200 NVSwitch variant of the transport.  Its schedule is
stated on the collective's own chunk layout (R6: chunk c belongs to rank c;
AR = RS then AG) with two multicast primitives:

* ``mred(r, c)``:  <r,c> := (+)_k <k,c>        (multimem.ld_reduce through the multicast
  alias: the switch reads every rank's copy and returns the reduction)
* ``mcast(r, c)``: <k,c> := <r,c> for every k  (multimem.st: one store lands in every copy)

ReduceScatter = mred(r, r) on every rank; AllGather = mcast(r, r); AllReduce = mred(r, r)
then mcast(r, r), where AR's "chunk r" is rank r's slice of a 16-byte-aligned partition
(reading R28: the partition does not change the result, every element is
reduced by exactly one rank).

The switch's association order is not specified, so the value pass folds in rank order
k = 0..N-1 exactly as the definition does (``definition.reduce_all``); floating-point
sums are therefore compared with the north_star tolerance, while int32 (wraparound),
max/min and exactly-representable inputs are bit-exact.

The routing rule (which calls the NVLS kernel takes; every other call runs the
algorithm's primitive plan) is restated in ``eligible``.
"""
from __future__ import annotations

from typing import Dict, List, Set, Tuple

import numpy as np

from .definition import reduce_all

ELT = {"int32": 4, "float32": 4, "float16": 2, "bfloat16": 2}


def schedule(coll: str, n: int) -> List[Tuple[str, int, int]]:
    """The NVLS primitive list (op, rank, chunk) in issue order."""
    mred = [("mred", r, r) for r in range(n)]
    mcast = [("mcast", r, r) for r in range(n)]
    return {"reducescatter": mred, "allgather": mcast, "allreduce": mred + mcast}[coll]


def ar_partition(nbytes: int, n: int) -> List[Tuple[int, int]]:
    """R28: rank r's AllReduce byte range [lo, hi): slices of ceil(S/N) rounded up to 16 B."""
    sl = ((nbytes + n - 1) // n + 15) // 16 * 16
    out = []
    for r in range(n):
        lo = min(r * sl, nbytes)
        out.append((lo, min(lo + sl, nbytes)))
    return out


def eligible(coll: str, count: int, dtype: str, op: str, send_off: int = 0, recv_off: int = 0) -> bool:
    """Routing rule (include/resccl.h, f3), for buffers inside NVLS windows at byte offsets
    send_off / recv_off: the offsets are 4-byte aligned, each rank's block is whole 4-byte
    granules and the op has a multimem.ld_reduce form (float32 has add only)."""
    if dtype == "float32" and op != "sum":
        return False
    return (count * ELT[dtype]) % 4 == 0 and send_off % 4 == 0 and recv_off % 4 == 0


def symbolic(coll: str, n: int) -> Dict[Tuple[int, int], Set[int]]:
    """Symbolic replay (extended to mred/mcast): every location holds the
    set of ranks contributing to it.  Raises on a non-disjoint reduction (I1) or a read of
    an undefined location (I6); the caller checks I3 on the result."""
    st: Dict[Tuple[int, int], Set[int]] = {}
    for r in range(n):
        for c in range(n):
            if coll == "allgather":
                if c == r:
                    st[(r, c)] = {r}
            else:
                st[(r, c)] = {r}
    for op, r, c in schedule(coll, n):
        if op == "mred":
            acc: Set[int] = set()
            for k in range(n):
                src = st.get((k, c))
                if src is None:
                    raise AssertionError(f"mred reads undefined <{k},{c}>")
                if acc & src:
                    raise AssertionError(f"mred({r},{c}): contributions overlap")
                acc |= src
            st[(r, c)] = acc
        else:
            src = st.get((r, c))
            if src is None:
                raise AssertionError(f"mcast reads undefined <{r},{c}>")
            for k in range(n):
                st[(k, c)] = set(src)
    return st


def replay(coll: str, sends: List[np.ndarray], dtype: str, op: str = "sum") -> List[np.ndarray]:
    """Value pass of the schedule over per-rank host buffers (out-of-place: a location
    before its first write is read from sendbuf).  AR/RS: sends[k] holds count / N*count
    elements; AG: sends[k] holds the rank's block."""
    n = len(sends)
    if coll == "allgather":
        cnt = sends[0].size
        recvs = [np.zeros(n * cnt, dtype=sends[0].dtype) for _ in range(n)]
        for _, r, c in schedule(coll, n):  # mcast(r, r)
            for k in range(n):
                recvs[k][c * cnt:(c + 1) * cnt] = sends[r]
        return recvs
    if coll == "reducescatter":
        cnt = sends[0].size // n
        recvs = [np.zeros(cnt, dtype=sends[0].dtype) for _ in range(n)]
        for _, r, c in schedule(coll, n):  # mred(r, r)
            recvs[r][:] = reduce_all([s[c * cnt:(c + 1) * cnt] for s in sends], dtype, op)
        return recvs
    e = ELT[dtype]
    parts = ar_partition(sends[0].size * e, n)
    recvs = [np.zeros_like(s) for s in sends]
    for kind, r, c in schedule(coll, n):
        lo, hi = parts[c][0] // e, parts[c][1] // e
        if kind == "mred":
            recvs[r][lo:hi] = reduce_all([s[lo:hi] for s in sends], dtype, op)
        else:
            for k in range(n):
                recvs[k][lo:hi] = recvs[r][lo:hi]
    return recvs
