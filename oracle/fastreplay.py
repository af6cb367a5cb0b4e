"""Oracle: ctypes front of the C++17 fast schedule replay (``fastreplay.cc``, SURVEY §8(c)
c6).  TEST INFRASTRUCTURE ONLY.

``replay_full(ir, inputs, dtype, count, threads)`` returns every rank's receive buffer
for full-size inputs (numpy arrays in the storage layout of ``resccl_inputs``: bfloat16
as uint16 bit patterns).  Same result as ``replay.dataflow_values`` / ``replay.replay``
(pinned in tests/test_oracle_fast.py); sum only.

The library is built by ``__graft_entry__.build()`` (``build_lib()`` below): g++ only,
no CUDA headers.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import List

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "fastreplay.cc")
LIB = os.path.join(HERE, "liboracle_fastreplay.so")
DT = {"int32": 0, "float32": 1, "float16": 2, "bfloat16": 3}
STORE = {"int32": np.int32, "float32": np.float32, "float16": np.float16, "bfloat16": np.uint16}
_lib = None


def build_lib(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = f"{LIB}.{os.getpid()}.tmp"   # concurrent builders (pytest -n) never see a partial file
        subprocess.run(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-Wall", SRC, "-o", tmp],
                       check=True)
        os.replace(tmp, LIB)
    return LIB


def _load():
    global _lib
    if _lib is None:
        build_lib()
        _lib = ctypes.CDLL(LIB)
        _lib.oracle_fast_replay.restype = ctypes.c_int
        _lib.oracle_fast_replay.argtypes = [ctypes.c_char_p, ctypes.c_int, ctypes.POINTER(ctypes.c_void_p),
                                            ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_void_p),
                                            ctypes.c_longlong, ctypes.c_int]
    return _lib


def replay_full(ir, inputs: List[np.ndarray], dtype: str, count: int, threads: int = 1,
                outputs: List[np.ndarray] = None, work: List[np.ndarray] = None) -> List[np.ndarray]:
    """``ir``: an oracle IR (``oracle.ir.IR``) or IR text.  ``inputs[r]``: rank r's send
    buffer.  ``outputs``: optional preallocated receive buffers (AR: may be the inputs
    themselves, in place); ``work`` (ReduceScatter): optional preallocated N x count
    location buffers (timing loops reuse both, so first-touch page faults stay out)."""
    lib = _load()
    text = ir if isinstance(ir, str) else ir.to_text()
    n = len(inputs)
    coll = [ln for ln in text.splitlines() if ln.startswith("algo ")][0].split("coll=")[1].split()[0]
    st = STORE[dtype]
    ins = [np.ascontiguousarray(x, dtype=st) for x in inputs]
    if outputs is None:
        m = count * n if coll == "allgather" else count
        outputs = [np.empty(m, dtype=st) for _ in range(n)]
    if coll == "reducescatter" and work is None:
        work = [np.empty(n * count, dtype=st) for _ in range(n)]
    elif coll != "reducescatter":
        work = None
    P = ctypes.c_void_p * n
    sp = P(*[x.ctypes.data for x in ins])
    rp = P(*[y.ctypes.data for y in outputs])
    wp = P(*[w.ctypes.data for w in work]) if work else None
    rc = lib.oracle_fast_replay(text.encode(), DT[dtype], sp, rp, wp, count, threads)
    if rc != 0:
        raise ValueError(f"oracle_fast_replay failed ({rc})")
    return outputs
