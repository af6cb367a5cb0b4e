"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds ONLY the input recipe; none of the
collective's arithmetic lives here.  Both sides of every parity check (the CPU
oracle under ``oracle/`` and the CUDA path under
``paper_conf_sigcomm_liuhlgcwz025_b200``) receive the arrays produced here.

Recipe (per rank ``r``, element ``i``)::

    x = splitmix64(seed ^ (r << 32) ^ i)

* ``int32``    uniform in [-2^20, 2^20)  (no overflow when summed over <= 2^11 ranks)
  ``int32_wrap`` full 32-bit range (exercises two's-complement wraparound)
* ``float32``  k / 2^23 for k uniform in [-2^23, 2^23)  -> uniform [-1, 1), exact
* ``float16``  k / 2^10 for k uniform in [-2^10, 2^10)  -> uniform [-1, 1), exact
* ``bfloat16`` upper 16 bits of the float32 draw (truncation, no rounding) -> [-1, 1)
* ``exact`` mode: integers in [-4, 4] for every dtype, so every partial sum of
  <= 8 ranks is exactly representable in bf16/fp16/fp32 (order-free results).

bfloat16 values are carried as ``numpy.uint16`` bit patterns.
"""
from __future__ import annotations

import numpy as np

DTYPES = ("int32", "float32", "float16", "bfloat16")
ELEM_SIZE = {"int32": 4, "float32": 4, "float16": 2, "bfloat16": 2}
NP_STORAGE = {"int32": np.int32, "float32": np.float32, "float16": np.float16,
              "bfloat16": np.uint16}

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser (Steele et al.); input/output uint64."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)) & _M64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _M64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _M64
        return z ^ (z >> np.uint64(31))


def raw_bits(seed: int, rank: int, n: int, offset: int = 0) -> np.ndarray:
    idx = np.arange(offset, offset + n, dtype=np.uint64)
    key = np.uint64((seed & 0xFFFFFFFF) ^ ((rank & 0xFFFFFFFF) << 32))
    return splitmix64(idx ^ key)


def rank_input(dtype: str, seed: int, rank: int, n: int, mode: str = "uniform",
               offset: int = 0) -> np.ndarray:
    """Input vector of ``n`` elements for ``rank`` (elements ``offset..offset+n``)."""
    z = raw_bits(seed, rank, n, offset)
    if mode == "exact":
        k = (z % np.uint64(9)).astype(np.int64) - 4          # [-4, 4]
        if dtype == "int32":
            return k.astype(np.int32)
        if dtype == "float32":
            return k.astype(np.float32)
        if dtype == "float16":
            return k.astype(np.float16)
        if dtype == "bfloat16":
            # small integers are exact in bf16: take the fp32 bit pattern's top half
            return (k.astype(np.float32).view(np.uint32) >> np.uint32(16)).astype(np.uint16)
        raise ValueError(dtype)
    if mode == "wrap":
        assert dtype == "int32"
        return (z >> np.uint64(32)).astype(np.uint32).view(np.int32)
    if mode != "uniform":
        raise ValueError(mode)
    if dtype == "int32":
        return ((z >> np.uint64(43)).astype(np.int64) - (1 << 20)).astype(np.int32)
    if dtype == "float32":
        k = (z >> np.uint64(40)).astype(np.int64) - (1 << 23)
        return (k.astype(np.float64) / float(1 << 23)).astype(np.float32)
    if dtype == "float16":
        k = (z >> np.uint64(53)).astype(np.int64) - (1 << 10)
        return (k.astype(np.float64) / float(1 << 10)).astype(np.float16)
    if dtype == "bfloat16":
        k = (z >> np.uint64(40)).astype(np.int64) - (1 << 23)
        f = (k.astype(np.float64) / float(1 << 23)).astype(np.float32)
        return (f.view(np.uint32) >> np.uint32(16)).astype(np.uint16)
    raise ValueError(dtype)


def all_inputs(dtype: str, seed: int, nranks: int, n: int, mode: str = "uniform"):
    return [rank_input(dtype, seed, r, n, mode) for r in range(nranks)]
