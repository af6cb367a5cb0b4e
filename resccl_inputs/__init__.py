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


def rank_input_at(dtype: str, seed: int, rank: int, idx: np.ndarray, mode: str = "uniform") -> np.ndarray:
    """Same recipe at arbitrary element positions ``idx`` (for sampled full-size checks)."""
    idx = np.asarray(idx, dtype=np.uint64)
    key = np.uint64((seed & 0xFFFFFFFF) ^ ((rank & 0xFFFFFFFF) << 32))
    return _from_bits(splitmix64(idx ^ key), dtype, mode)


def _from_bits(z, dtype, mode):
    if mode == "exact":
        k = (z % np.uint64(9)).astype(np.int64) - 4
        if dtype == "bfloat16":
            return (k.astype(np.float32).view(np.uint32) >> np.uint32(16)).astype(np.uint16)
        return k.astype(NP_STORAGE[dtype])
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


def rank_input_torch(dtype: str, seed: int, rank: int, n: int, device="cuda:0", mode: str = "uniform",
                     block: int = 1 << 26):
    """The same recipe evaluated with torch on ``device`` (for full-size buffers whose
    host generation would be too slow).  Bit-identical to ``rank_input`` (pinned by
    tests/test_inputs.py)."""
    import torch
    tdt = {"int32": torch.int32, "float32": torch.float32, "float16": torch.float16,
           "bfloat16": torch.bfloat16}[dtype]
    out = torch.empty(n, dtype=tdt, device=device)
    M32 = 0xFFFFFFFF
    key = (seed & M32) ^ ((rank & M32) << 32)
    if key >= 1 << 63:
        key -= 1 << 64

    def srl(x, k):  # logical right shift of int64
        return (x >> k) & ((1 << (64 - k)) - 1)

    def s64(c):
        return c - (1 << 64) if c >= 1 << 63 else c

    for lo in range(0, n, block):
        hi = min(n, lo + block)
        x = torch.arange(lo, hi, dtype=torch.int64, device=device) ^ key
        z = x + s64(0x9E3779B97F4A7C15)
        z = (z ^ srl(z, 30)) * s64(0xBF58476D1CE4E5B9)
        z = (z ^ srl(z, 27)) * s64(0x94D049BB133111EB)
        z = z ^ srl(z, 31)
        if mode == "exact":
            # unsigned z mod 9 from the signed representation
            k = (((srl(z, 32) % 9) * (2 ** 32 % 9) + (z & M32) % 9) % 9) - 4
            v = k.to(torch.float32).to(tdt) if dtype != "int32" else k.to(torch.int32)
        elif dtype == "int32":
            v = (srl(z, 43) - (1 << 20)).to(torch.int32)
        elif dtype == "float16":
            v = ((srl(z, 53) - (1 << 10)).to(torch.float64) / float(1 << 10)).to(torch.float16)
        else:
            f = ((srl(z, 40) - (1 << 23)).to(torch.float64) / float(1 << 23)).to(torch.float32)
            if dtype == "bfloat16":
                v = (f.view(torch.int32) >> 16).to(torch.int16).view(torch.bfloat16)
            else:
                v = f
        out[lo:hi] = v
    return out
