"""Oracle: element arithmetic of the collectives.  TEST INFRASTRUCTURE ONLY.

Reading R8: one combine step is ``local (+) incoming``; bf16/fp16
operands are widened to binary32, combined in binary32 and rounded back to the
storage type with round-to-nearest-even at every store or forward; fp32 is native
binary32; int32 wraps (two's complement).  No flush-to-zero.  The reduction op
is sum (the paper's only op), with max/min as optional extras (R17).

bfloat16 values are uint16 bit patterns.
"""
from __future__ import annotations

import numpy as np


def bf16_to_f32(u16: np.ndarray) -> np.ndarray:
    return (u16.astype(np.uint32) << np.uint32(16)).view(np.float32)


def f32_to_bf16_rne(f: np.ndarray) -> np.ndarray:
    """IEEE round-to-nearest-even of binary32 to bfloat16 (NaN inputs not expected)."""
    b = np.ascontiguousarray(f, dtype=np.float32).view(np.uint32).astype(np.uint64)
    lsb = (b >> np.uint64(16)) & np.uint64(1)
    r = (b + np.uint64(0x7FFF) + lsb) >> np.uint64(16)
    return r.astype(np.uint16)


def f64_to_f32_round_to_odd(d: np.ndarray) -> np.ndarray:
    """binary64 -> binary32 with round-to-odd (truncate toward zero, then set the
    last bit if inexact).  Rounding to odd at >= p+2 bits followed by RNE to p bits
    equals a single RNE to p bits (Boldo & Melquiond), so binary64 -> bf16/fp16 is
    correctly rounded without double rounding."""
    d = np.asarray(d, dtype=np.float64)
    f = d.astype(np.float32)
    back = f.astype(np.float64)
    inexact = back != d
    toward0 = np.abs(back) > np.abs(d)
    f = np.where(inexact & toward0, np.nextafter(f, np.float32(0)), f).astype(np.float32)
    bits = f.view(np.uint32).copy()
    bits[inexact] |= np.uint32(1)
    return bits.view(np.float32)


def f64_to_dtype_rne(d: np.ndarray, dtype: str) -> np.ndarray:
    """Single correctly-rounded (RNE) conversion of binary64 values to ``dtype``."""
    if dtype == "float32":
        return np.asarray(d, dtype=np.float64).astype(np.float32)
    f = f64_to_f32_round_to_odd(d)
    if dtype == "bfloat16":
        return f32_to_bf16_rne(f)
    if dtype == "float16":
        return f.astype(np.float16)
    raise ValueError(dtype)


def f64_to_bf16_scalar(x: float) -> int:
    """Independent scalar RNE binary64 -> bfloat16 (frexp-based), used only to pin
    the vectorised round-to-odd path above."""
    import math
    if x == 0.0:
        return 0x8000 if math.copysign(1.0, x) < 0 else 0
    sign = 0x8000 if x < 0 else 0
    a = abs(x)
    m, e = math.frexp(a)           # a = m * 2^e, m in [0.5, 1)
    quantum = 2.0 ** -133 if e - 1 < -126 else 2.0 ** (e - 1 - 7)
    q = a / quantum
    fl = math.floor(q)
    rem = q - fl
    if rem > 0.5 or (rem == 0.5 and (fl % 2 == 1)):
        fl += 1
    f32 = np.float32(fl * quantum)
    if not np.isfinite(f32):
        return sign | 0x7F80
    return sign | int(np.array([f32], dtype=np.float32).view(np.uint32)[0] >> 16)


def to_f32(x: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "bfloat16":
        return bf16_to_f32(x)
    return x.astype(np.float32)


def from_f32(f: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "bfloat16":
        return f32_to_bf16_rne(f)
    if dtype == "float16":
        return f.astype(np.float16)          # numpy rounds to nearest even
    if dtype == "float32":
        return f.astype(np.float32)
    raise ValueError(dtype)


def combine(local: np.ndarray, incoming: np.ndarray, dtype: str, op: str = "sum") -> np.ndarray:
    """One reduction step ``local (+) incoming`` with the storage-type rounding of R8."""
    if dtype == "int32":
        a = local.astype(np.int64)
        b = incoming.astype(np.int64)
        if op == "sum":
            return ((a + b) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
        if op == "max":
            return np.maximum(a, b).astype(np.int32)
        if op == "min":
            return np.minimum(a, b).astype(np.int32)
        raise ValueError(op)
    fa = to_f32(local, dtype)
    fb = to_f32(incoming, dtype)
    if op == "sum":
        r = (fa + fb).astype(np.float32)
    elif op == "max":
        r = np.maximum(fa, fb)
    elif op == "min":
        r = np.minimum(fa, fb)
    else:
        raise ValueError(op)
    return from_f32(r, dtype)
