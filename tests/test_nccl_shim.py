"""f4: the NCCL-symbol shim (libresccl_nccl.so, include/resccl_nccl.h) -- "relink and
rebuild".

CPU: the library exports the NCCL entry points the header declares, and its TCP
rendezvous (ncclGetUniqueId -> every rank's blob to every rank) works across 3
processes.  GPU: two processes bootstrap with ncclGetUniqueId / ncclCommInitRank and
run ncclAllReduce / ncclAllGather / ncclReduceScatter / ncclBroadcast on device
buffers; results equal the oracle's definitions bit for bit (int32, wraparound)."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SHIM = os.path.join(ROOT, "paper_conf_sigcomm_liuhlgcwz025_b200", "libresccl_nccl.so")
HDR = os.path.join(ROOT, "include", "resccl_nccl.h")


class UniqueId(ctypes.Structure):
    _fields_ = [("internal", ctypes.c_char * 128)]


def _lib():
    lib = ctypes.CDLL(SHIM)
    lib.ncclGetUniqueId.argtypes = [ctypes.POINTER(UniqueId)]
    lib.rescclShimExchange.argtypes = [ctypes.POINTER(UniqueId), ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                       ctypes.c_size_t, ctypes.c_void_p, ctypes.POINTER(ctypes.c_size_t),
                                       ctypes.POINTER(ctypes.c_size_t)]
    lib.ncclGetErrorString.restype = ctypes.c_char_p
    lib.ncclCommInitRank.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.c_int, UniqueId, ctypes.c_int]
    return lib


def test_shim_exports_every_declared_symbol():
    names = re.findall(r"^(?:ncclResult_t|const char\*)\s+(\w+)\(", open(HDR).read(), re.M)
    assert len(names) >= 18
    out = subprocess.run(["nm", "-D", "--defined-only", SHIM], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r" T (\w+)$", out, re.M))
    assert set(names) <= exported, set(names) - exported
    lib = _lib()
    v = ctypes.c_int(0)
    assert lib.ncclGetVersion(ctypes.byref(v)) == 0 and v.value >= 22000
    assert lib.ncclGetErrorString(4) == b"invalid argument (ResCCL)"


def _xchg_worker(rank, n, idb, q):
    try:
        lib = _lib()
        uid = UniqueId()
        ctypes.memmove(ctypes.addressof(uid), idb, 128)
        blob = bytes([rank + 1]) * (10 + rank)
        cap = ctypes.c_size_t(4096)
        out = ctypes.create_string_buffer(4096)
        lens = (ctypes.c_size_t * n)()
        rc = lib.rescclShimExchange(ctypes.byref(uid), rank, n, blob, len(blob), out, ctypes.byref(cap), lens)
        q.put((rank, rc, out.raw[:cap.value], list(lens)))
    except Exception as e:  # pragma: no cover
        q.put((rank, -1, repr(e), None))


@pytest.mark.timeout(120)
def test_shim_rendezvous_three_processes():
    import multiprocessing as mp
    lib = _lib()
    uid = UniqueId()
    assert lib.ncclGetUniqueId(ctypes.byref(uid)) == 0
    assert ctypes.string_at(ctypes.addressof(uid), 8) == b"RESCCLID"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    n = 3
    ps = [ctx.Process(target=_xchg_worker, args=(r, n, ctypes.string_at(ctypes.addressof(uid), 128), q)) for r in range(n)]
    for p in ps:
        p.start()
    res = [q.get(timeout=100) for _ in range(n)]
    for p in ps:
        p.join(20)
    want = b"".join(bytes([r + 1]) * (10 + r) for r in range(n))
    for rank, rc, blob, lens in res:
        assert rc == 0, blob
        assert blob == want and lens == [10 + r for r in range(n)]


def _gpu_worker(rank, n, idb, q):
    try:
        import sys
        sys.path.insert(0, ROOT)
        import torch
        import resccl_inputs as inp
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        torch.zeros(1, device="cuda")  # make the device's context current (NCCL's rule)
        lib = _lib()
        uid = UniqueId()
        ctypes.memmove(ctypes.addressof(uid), idb, 128)
        comm = ctypes.c_void_p()
        rc = lib.ncclCommInitRank(ctypes.byref(comm), n, uid, rank)
        assert rc == 0, rc
        s = torch.cuda.current_stream().cuda_stream
        cnt = 5003
        x = torch.from_numpy(inp.rank_input("int32", 8, rank, cnt, mode="wrap")).cuda()
        out = {}
        r = torch.empty_like(x)
        assert lib.ncclAllReduce(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(r.data_ptr()), ctypes.c_size_t(cnt),
                                 2, 0, comm, ctypes.c_void_p(s)) == 0
        out["ar"] = r.cpu().numpy()
        g = torch.empty(n * cnt, dtype=torch.int32, device="cuda")
        assert lib.ncclAllGather(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(g.data_ptr()), ctypes.c_size_t(cnt),
                                 2, comm, ctypes.c_void_p(s)) == 0
        out["ag"] = g.cpu().numpy()
        big = torch.from_numpy(inp.rank_input("int32", 9, rank, n * cnt, mode="wrap")).cuda()
        rs = torch.empty(cnt, dtype=torch.int32, device="cuda")
        assert lib.ncclReduceScatter(ctypes.c_void_p(big.data_ptr()), ctypes.c_void_p(rs.data_ptr()),
                                     ctypes.c_size_t(cnt), 2, 0, comm, ctypes.c_void_p(s)) == 0
        out["rs"] = rs.cpu().numpy()
        b = torch.from_numpy(inp.rank_input("float32", 10, rank, cnt)).cuda()
        bo = torch.empty_like(b)
        assert lib.ncclBroadcast(ctypes.c_void_p(b.data_ptr()), ctypes.c_void_p(bo.data_ptr()), ctypes.c_size_t(cnt),
                                 7, 1, comm, ctypes.c_void_p(s)) == 0
        out["bc"] = bo.cpu().numpy()
        assert lib.ncclAllReduce(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(r.data_ptr()), ctypes.c_size_t(cnt),
                                 2, 1, comm, ctypes.c_void_p(s)) == 4  # ncclProd -> invalid argument
        torch.cuda.synchronize()
        err = ctypes.c_int(-1)
        assert lib.ncclCommGetAsyncError(comm, ctypes.byref(err)) == 0 and err.value == 0
        assert lib.ncclCommDestroy(comm) == 0
        q.put((rank, out, None))
    except Exception:
        import traceback
        q.put((rank, None, traceback.format_exc()))


@pytest.mark.gpu
@pytest.mark.timeout(300)
def test_shim_collectives_two_processes():
    import torch.multiprocessing as mp
    import resccl_inputs as inp
    from oracle import definition
    lib = _lib()
    uid = UniqueId()
    assert lib.ncclGetUniqueId(ctypes.byref(uid)) == 0
    n, cnt = 2, 5003
    os.environ["RESCCL_TIMEOUT_MS"] = "60000"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_gpu_worker, args=(r, n, ctypes.string_at(ctypes.addressof(uid), 128), q)) for r in range(n)]
    for p in ps:
        p.start()
    res = {}
    for _ in range(n):
        rank, out, tb = q.get(timeout=280)
        assert tb is None, tb
        res[rank] = out
    for p in ps:
        p.join(30)
    xs = [inp.rank_input("int32", 8, r, cnt, mode="wrap") for r in range(n)]
    bigs = [inp.rank_input("int32", 9, r, n * cnt, mode="wrap") for r in range(n)]
    root = inp.rank_input("float32", 10, 1, cnt)
    ar, ag, rs = definition.allreduce(xs, "int32"), definition.allgather(xs), definition.reducescatter(bigs, "int32")
    for r in range(n):
        assert np.array_equal(res[r]["ar"], ar[r])
        assert np.array_equal(res[r]["ag"], ag[r])
        assert np.array_equal(res[r]["rs"], rs[r])
        assert np.array_equal(res[r]["bc"].view(np.uint32), root.view(np.uint32))
