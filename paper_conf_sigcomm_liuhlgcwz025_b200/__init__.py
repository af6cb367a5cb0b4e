"""B200-native ResCCL hot path: Python binding of the C ABI (include/resccl.h).

Argument marshalling only: every step of the path (planning, kernel generation,
transport) runs in ``libresccl.so`` and its NVRTC-compiled sm_100a kernels.  The
functions below carry the C ABI names.  PyTorch is used only for device memory,
streams and (optionally) process groups for the IPC-handle exchange.

If the native library is missing, importing this package raises -- there is no
CPU or PyTorch fallback.
"""
from __future__ import annotations

import ctypes
import json
import os
from typing import List, Optional, Sequence

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libresccl.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} not built; run `python -c 'import __graft_entry__ as g; g.build()'` "
        "(the ResCCL path has no fallback)")

_lib = ctypes.CDLL(LIB_PATH)

# ------------------------------------------------------------------ enums (resccl.h)
rescclSuccess, rescclInvalidArgument, rescclInvalidUsage, rescclCudaError, \
    rescclSystemError, rescclInternalError, rescclTimeout = range(7)
rescclInt32, rescclFloat32, rescclFloat16, rescclBfloat16 = range(4)
rescclSum, rescclMax, rescclMin = range(3)
rescclCollAllGather, rescclCollReduceScatter, rescclCollAllReduce = range(3)

DTYPES = {"int32": rescclInt32, "float32": rescclFloat32, "float16": rescclFloat16,
          "bfloat16": rescclBfloat16}
OPS = {"sum": rescclSum, "max": rescclMax, "min": rescclMin}
COLLS = {"allgather": rescclCollAllGather, "reducescatter": rescclCollReduceScatter,
         "allreduce": rescclCollAllReduce}

EXPORTS = [
    "rescclGetErrorString", "rescclGetLastError", "rescclGetVersion", "rescclCommCreate",
    "rescclCommGetHandle", "rescclCommConnect", "rescclCommInit", "rescclCommInitAll",
    "rescclCommDestroy", "rescclCommRank", "rescclCommCount", "rescclCommCuDevice", "rescclCommGetAsyncError",
    "rescclLoadAlgorithm", "rescclSetActiveAlgorithm", "rescclGetPlanInfo", "rescclGetTbUtilization",
    "rescclGetPhaseTrace",
    "rescclAllReduce",
    "rescclAllGather", "rescclReduceScatter", "rescclGenerateIr", "rescclPlanIr",
    "rescclCodegenIr", "rescclCompileIr", "rescclCheckDeadlock", "rescclParseResCCLang", "rescclProfilePlanner",
    "rescclCommRegister", "rescclCommRegisterConnect", "rescclSimulateTimeline",
    "rescclNvlsSupported", "rescclNvlsAlloc", "rescclNvlsAllocAll", "rescclNvlsFree", "rescclCompileNvls",
]

_c = ctypes
_vp, _sz, _i = _c.c_void_p, _c.c_size_t, _c.c_int
_SIGS = {
    "rescclGetErrorString": (_c.c_char_p, [_i]),
    "rescclGetLastError": (_c.c_char_p, []),
    "rescclGetVersion": (_i, []),
    "rescclCommCreate": (_i, [_i, _i, _i, _c.POINTER(_vp)]),
    "rescclCommGetHandle": (_i, [_vp, _vp, _c.POINTER(_sz)]),
    "rescclCommConnect": (_i, [_vp, _c.POINTER(_vp), _c.POINTER(_sz)]),
    "rescclCommInitAll": (_i, [_c.POINTER(_vp), _i, _c.POINTER(_i)]),
    "rescclCommDestroy": (_i, [_vp]),
    "rescclCommRank": (_i, [_vp, _c.POINTER(_i)]),
    "rescclCommCount": (_i, [_vp, _c.POINTER(_i)]),
    "rescclCommCuDevice": (_i, [_vp, _c.POINTER(_i)]),
    "rescclCommGetAsyncError": (_i, [_vp, _c.POINTER(_i)]),
    "rescclLoadAlgorithm": (_i, [_vp, _c.c_char_p, _c.POINTER(_vp)]),
    "rescclSetActiveAlgorithm": (_i, [_vp, _vp]),
    "rescclGetPlanInfo": (_i, [_vp, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclGetTbUtilization": (_i, [_vp, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclGetPhaseTrace": (_i, [_vp, _vp, _c.POINTER(_sz)]),
    "rescclAllReduce": (_i, [_vp, _vp, _sz, _i, _i, _vp, _vp]),
    "rescclAllGather": (_i, [_vp, _vp, _sz, _i, _vp, _vp]),
    "rescclReduceScatter": (_i, [_vp, _vp, _sz, _i, _i, _vp, _vp]),
    "rescclGenerateIr": (_i, [_c.c_char_p, _i, _i, _c.c_char_p, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclPlanIr": (_i, [_c.c_char_p, _c.c_char_p, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclSimulateTimeline": (_i, [_c.c_char_p, _c.c_char_p, _c.c_char_p, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclCodegenIr": (_i, [_c.c_char_p, _c.c_char_p, _i, _i, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclCompileIr": (_i, [_c.c_char_p, _c.c_char_p, _i, _i, _c.POINTER(_sz)]),
    "rescclCheckDeadlock": (_i, [_c.c_char_p, _c.c_char_p, _i, _i, _c.POINTER(_i)]),
    "rescclParseResCCLang": (_i, [_c.c_char_p, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclProfilePlanner": (_i, [_c.c_char_p, _c.c_char_p, _i, _c.c_char_p, _c.POINTER(_sz)]),
    "rescclCommRegister": (_i, [_vp, _vp, _sz, _vp, _c.POINTER(_sz)]),
    "rescclCommRegisterConnect": (_i, [_vp, _c.POINTER(_vp), _c.POINTER(_sz), _c.POINTER(_i)]),
    "rescclNvlsSupported": (_i, [_vp, _c.POINTER(_i)]),
    "rescclNvlsAlloc": (_i, [_vp, _sz, _vp, _vp, _c.POINTER(_vp)]),
    "rescclNvlsAllocAll": (_i, [_c.POINTER(_vp), _i, _sz, _c.POINTER(_vp)]),
    "rescclNvlsFree": (_i, [_vp, _vp]),
    "rescclCompileNvls": (_i, [_i, _i, _i, _c.POINTER(_sz)]),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


class ResCCLError(RuntimeError):
    def __init__(self, code: int, where: str):
        msg = _lib.rescclGetLastError().decode(errors="replace")
        super().__init__(f"{where}: {_lib.rescclGetErrorString(code).decode()} ({code}): {msg}")
        self.code = code


def _check(code: int, where: str):
    if code != rescclSuccess:
        raise ResCCLError(code, where)


def _b(s):
    return s.encode() if isinstance(s, str) else s


def _sized(fn, *args) -> str:
    n = _sz(0)
    _check(fn(*args, None, _c.byref(n)), fn.__name__)
    for _ in range(4):  # outputs with timings may grow between the two calls
        cap = n.value + 4096
        buf = _c.create_string_buffer(cap)
        n = _sz(cap)
        rc = fn(*args, buf, _c.byref(n))
        if rc == rescclInvalidArgument and n.value > cap:
            continue
        _check(rc, fn.__name__)
        return buf.value.decode()
    _check(rc, fn.__name__)


# ------------------------------------------------------------------ C-ABI wrappers (same names)

def rescclGetErrorString(code: int) -> str:
    return _lib.rescclGetErrorString(code).decode()


def rescclGetLastError() -> str:
    return _lib.rescclGetLastError().decode()


def rescclGetVersion() -> int:
    return _lib.rescclGetVersion()


def rescclCommCreate(rank: int, nranks: int, device: int) -> int:
    out = _vp()
    _check(_lib.rescclCommCreate(rank, nranks, device, _c.byref(out)), "rescclCommCreate")
    return out.value


def rescclCommGetHandle(comm: int) -> bytes:
    n = _sz(0)
    _check(_lib.rescclCommGetHandle(comm, None, _c.byref(n)), "rescclCommGetHandle")
    buf = _c.create_string_buffer(n.value)
    _check(_lib.rescclCommGetHandle(comm, _c.cast(buf, _vp), _c.byref(n)), "rescclCommGetHandle")
    return buf.raw[:n.value]


def rescclCommConnect(comm: int, handles: Sequence[bytes]) -> None:
    bufs = [_c.create_string_buffer(h, len(h)) for h in handles]
    arr = (_vp * len(bufs))(*[_c.cast(b, _vp) for b in bufs])
    lens = (_sz * len(bufs))(*[len(h) for h in handles])
    _check(_lib.rescclCommConnect(comm, arr, lens), "rescclCommConnect")


def rescclCommInitAll(devices: Sequence[int]) -> List[int]:
    n = len(devices)
    comms = (_vp * n)()
    devs = (_i * n)(*devices)
    _check(_lib.rescclCommInitAll(comms, n, devs), "rescclCommInitAll")
    return [comms[k] for k in range(n)]


def rescclCommRegister(comm: int, ptr: int, nbytes: int) -> bytes:
    n = _sz(0)
    _check(_lib.rescclCommRegister(comm, ptr, nbytes, None, _c.byref(n)), "rescclCommRegister")
    buf = _c.create_string_buffer(n.value)
    _check(_lib.rescclCommRegister(comm, ptr, nbytes, _c.cast(buf, _vp), _c.byref(n)), "rescclCommRegister")
    return buf.raw[:n.value]


def rescclCommRegisterConnect(comm: int, blobs: Sequence[bytes]) -> int:
    bufs = [_c.create_string_buffer(h, len(h)) for h in blobs]
    arr = (_vp * len(bufs))(*[_c.cast(b, _vp) for b in bufs])
    lens = (_sz * len(bufs))(*[len(h) for h in blobs])
    w = _i()
    _check(_lib.rescclCommRegisterConnect(comm, arr, lens, _c.byref(w)), "rescclCommRegisterConnect")
    return w.value


# allgather callback of rescclCommInit / rescclNvlsAlloc: int (*)(const void*, void*, size_t, void*)
ALLGATHER_CB = _c.CFUNCTYPE(_i, _vp, _vp, _sz, _vp)


def rescclNvlsSupported(comm: int) -> bool:
    v = _i()
    _check(_lib.rescclNvlsSupported(comm, _c.byref(v)), "rescclNvlsSupported")
    return bool(v.value)


def rescclNvlsAlloc(comm: int, nbytes: int, allgather) -> int:
    """Multi-process NVLS window (collective).  `allgather(data: bytes) -> List[bytes]`
    gathers one equal-length blob from every rank, rank-major."""
    def cb(inp, out, n, _ctx):
        try:
            parts = allgather(_c.string_at(inp, n))
            joined = b"".join(parts)
            _c.memmove(out, joined, len(joined))
            return 0
        except Exception:  # noqa: BLE001 -- reported through the C ABI as a SystemError
            return 1
    fn = ALLGATHER_CB(cb)
    p = _vp()
    _check(_lib.rescclNvlsAlloc(comm, nbytes, _c.cast(fn, _vp), None, _c.byref(p)), "rescclNvlsAlloc")
    return p.value


def rescclNvlsAllocAll(comms: Sequence[int], nbytes: int) -> List[int]:
    n = len(comms)
    arr = (_vp * n)(*comms)
    ptrs = (_vp * n)()
    _check(_lib.rescclNvlsAllocAll(arr, n, nbytes, ptrs), "rescclNvlsAllocAll")
    return [ptrs[k] for k in range(n)]


def rescclNvlsFree(comm: int, ptr: int) -> None:
    _check(_lib.rescclNvlsFree(comm, ptr), "rescclNvlsFree")


def rescclCompileNvls(coll: str, dtype: str = "bfloat16", op: str = "sum") -> int:
    n = _sz(0)
    _check(_lib.rescclCompileNvls(COLLS[coll], DTYPES[dtype], OPS[op], _c.byref(n)), "rescclCompileNvls")
    return n.value


def rescclCommDestroy(comm: int) -> None:
    _check(_lib.rescclCommDestroy(comm), "rescclCommDestroy")


def rescclCommRank(comm: int) -> int:
    r = _i()
    _check(_lib.rescclCommRank(comm, _c.byref(r)), "rescclCommRank")
    return r.value


def rescclCommCount(comm: int) -> int:
    r = _i()
    _check(_lib.rescclCommCount(comm, _c.byref(r)), "rescclCommCount")
    return r.value


def rescclCommGetAsyncError(comm: int) -> int:
    r = _i()
    _check(_lib.rescclCommGetAsyncError(comm, _c.byref(r)), "rescclCommGetAsyncError")
    return r.value


def rescclLoadAlgorithm(comm: int, ir_text: str) -> int:
    out = _vp()
    _check(_lib.rescclLoadAlgorithm(comm, _b(ir_text), _c.byref(out)), "rescclLoadAlgorithm")
    return out.value


def rescclSetActiveAlgorithm(comm: int, algo: int) -> None:
    _check(_lib.rescclSetActiveAlgorithm(comm, algo), "rescclSetActiveAlgorithm")


def rescclGetPlanInfo(algo: int) -> dict:
    n = _sz(0)
    _check(_lib.rescclGetPlanInfo(algo, None, _c.byref(n)), "rescclGetPlanInfo")
    buf = _c.create_string_buffer(n.value)
    _check(_lib.rescclGetPlanInfo(algo, buf, _c.byref(n)), "rescclGetPlanInfo")
    return json.loads(buf.value.decode())


def rescclGetTbUtilization(algo: int) -> dict:
    n = _sz(0)
    _check(_lib.rescclGetTbUtilization(algo, None, _c.byref(n)), "rescclGetTbUtilization")
    buf = _c.create_string_buffer(n.value)
    _check(_lib.rescclGetTbUtilization(algo, buf, _c.byref(n)), "rescclGetTbUtilization")
    return json.loads(buf.value.decode())


def rescclGetPhaseTrace(algo: int) -> List[int]:
    """Raw u64 words of the last launch's phase records (layout: include/resccl.h)."""
    n = _sz(0)
    _check(_lib.rescclGetPhaseTrace(algo, None, _c.byref(n)), "rescclGetPhaseTrace")
    buf = (_c.c_ulonglong * (n.value // 8))()
    _check(_lib.rescclGetPhaseTrace(algo, buf, _c.byref(n)), "rescclGetPhaseTrace")
    return list(buf)


def rescclAllReduce(sendbuf: int, recvbuf: int, count: int, dtype: int, op: int, comm: int,
                    stream: int = 0) -> None:
    _check(_lib.rescclAllReduce(sendbuf, recvbuf, count, dtype, op, comm, stream), "rescclAllReduce")


def rescclAllGather(sendbuf: int, recvbuf: int, sendcount: int, dtype: int, comm: int,
                    stream: int = 0) -> None:
    _check(_lib.rescclAllGather(sendbuf, recvbuf, sendcount, dtype, comm, stream), "rescclAllGather")


def rescclReduceScatter(sendbuf: int, recvbuf: int, recvcount: int, dtype: int, op: int, comm: int,
                        stream: int = 0) -> None:
    _check(_lib.rescclReduceScatter(sendbuf, recvbuf, recvcount, dtype, op, comm, stream),
           "rescclReduceScatter")


def rescclGenerateIr(name: str, coll: str, nranks: int, opts: str = "") -> str:
    return _sized(_lib.rescclGenerateIr, _b(name), COLLS[coll], nranks, _b(opts))


def rescclParseResCCLang(program: str) -> str:
    return _sized(_lib.rescclParseResCCLang, _b(program))


def rescclProfilePlanner(program: str, opts: str = "", verify: bool = False) -> dict:
    return json.loads(_sized(_lib.rescclProfilePlanner, _b(program), _b(opts), int(verify)))


def rescclPlanIr(ir_text: str, opts: str = "") -> dict:
    return json.loads(_sized(_lib.rescclPlanIr, _b(ir_text), _b(opts)))


def rescclSimulateTimeline(ir_text: str, opts: str = "", count: int = 1 << 20, elt: int = 2,
                           alpha: float = 2e-6, beta: float = 1 / 900e9, gamma: float = 2e-6) -> dict:
    params = f"count={count} elt={elt} alpha={alpha!r} beta={beta!r} gamma={gamma!r}"
    return json.loads(_sized(_lib.rescclSimulateTimeline, _b(ir_text), _b(opts), _b(params)))


def rescclCodegenIr(ir_text: str, opts: str = "", rank_lo: int = 0, rank_hi: Optional[int] = None) -> str:
    if rank_hi is None:
        rank_hi = int(ir_text.split("nranks=")[1].split()[0])
    return _sized(_lib.rescclCodegenIr, _b(ir_text), _b(opts), rank_lo, rank_hi)


def rescclCompileIr(ir_text: str, opts: str = "", dtype: int = rescclFloat32, op: int = rescclSum) -> int:
    n = _sz(0)
    _check(_lib.rescclCompileIr(_b(ir_text), _b(opts), dtype, op, _c.byref(n)), "rescclCompileIr")
    return n.value


def rescclCheckDeadlock(ir_text: str, opts: str = "", K: int = 1, n_mb: int = 2) -> bool:
    ok = _i()
    _check(_lib.rescclCheckDeadlock(_b(ir_text), _b(opts), K, n_mb, _c.byref(ok)), "rescclCheckDeadlock")
    return bool(ok.value)


from .torch_api import Communicator, VirtualGroup, init_process_group_comm  # noqa: E402,F401
