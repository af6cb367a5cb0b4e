"""Oracle: the collectives' definitions (c1).  TEST INFRASTRUCTURE ONLY.

AllGather, ReduceScatter and AllReduce are the operators named in P:L436-438;
AllReduce = ReduceScatter followed by AllGather.  The method only
makes these faster; their results are fixed by the definitions:

* AR: out_r[i] = (+)_{k=0}^{N-1} in_k[i] for every rank r
* AG: out_r[k*cnt + i] = in_k[i]
* RS: out_r[i] = (+)_k in_k[r*cnt + i]

(+) = sum: int32 wraps (computed in uint32); fp32 is the naive left fold
k = 0..N-1 in binary32; bf16/fp16 fold in binary64 and round once (RNE), the most
accurate reference for tolerance checks.  max/min (R17) are
order-free.
"""
from __future__ import annotations

from typing import List

import numpy as np

from .numerics import f64_to_dtype_rne, to_f32


def reduce_all(inputs: List[np.ndarray], dtype: str, op: str = "sum") -> np.ndarray:
    n = len(inputs)
    if dtype == "int32":
        acc = inputs[0].astype(np.int64)
        for k in range(1, n):
            x = inputs[k].astype(np.int64)
            if op == "sum":
                acc = (acc + x) & 0xFFFFFFFF
            elif op == "max":
                acc = np.maximum(acc, x)
            else:
                acc = np.minimum(acc, x)
        if op == "sum":
            return acc.astype(np.uint32).view(np.int32)
        return acc.astype(np.int32)
    if op in ("max", "min"):
        f = np.stack([to_f32(x, dtype) for x in inputs])
        r = f.max(axis=0) if op == "max" else f.min(axis=0)
        return _back(r, dtype)
    if dtype == "float32":
        acc = inputs[0].astype(np.float32)
        for k in range(1, n):
            acc = (acc + inputs[k].astype(np.float32)).astype(np.float32)
        return acc
    acc = to_f32(inputs[0], dtype).astype(np.float64)
    for k in range(1, n):
        acc = acc + to_f32(inputs[k], dtype).astype(np.float64)
    return f64_to_dtype_rne(acc, dtype)


def _back(f32: np.ndarray, dtype: str) -> np.ndarray:
    # max/min of exactly-representable values is exact in any storage type
    if dtype == "float32":
        return f32.astype(np.float32)
    return f64_to_dtype_rne(f32.astype(np.float64), dtype)


def allreduce(inputs: List[np.ndarray], dtype: str, op: str = "sum") -> List[np.ndarray]:
    r = reduce_all(inputs, dtype, op)
    return [r.copy() for _ in inputs]


def allgather(inputs: List[np.ndarray]) -> List[np.ndarray]:
    cat = np.concatenate(inputs)
    return [cat.copy() for _ in inputs]


def reducescatter(inputs: List[np.ndarray], dtype: str, op: str = "sum") -> List[np.ndarray]:
    n = len(inputs)
    cnt = inputs[0].size // n
    r = reduce_all(inputs, dtype, op)
    return [r[k * cnt:(k + 1) * cnt].copy() for k in range(n)]


def abs_sum(inputs: List[np.ndarray], dtype: str) -> np.ndarray:
    """sum_k |x_k[i]| in binary64 (denominator of the cancellation-safe tolerance)."""
    acc = np.zeros(inputs[0].shape, dtype=np.float64)
    for x in inputs:
        acc += np.abs(to_f32(x, dtype).astype(np.float64)) if dtype != "int32" else np.abs(x)
    return acc
