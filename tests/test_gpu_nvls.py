"""f3 (NVLS transport) on the GPU.

* Window allocation: on a multicast-capable fabric the NVLS kernel runs and is compared
  with the oracle's NVLS replay (oracle/nvls.py); where the driver refuses multicast (the
  gpurun boxes: one GPU alone in its NVLink partition, cuMulticastCreate ->
  CUDA_ERROR_INVALID_VALUE, profiles/r01_nvls_probe.txt) the error must come back cleanly
  through the C ABI and the parity part is skipped with that reason.
* Routing: an algorithm loaded with nvls=1 runs its primitive plan for every call that
  is not NVLS-eligible (virtual ranks, buffers outside windows) -- bit-exact vs the oracle.
* Multi-process allocation protocol: every rank makes the same callback calls whatever
  fails locally, so a refusal on one rank is an error on all ranks, never a hang.
"""
import os
import socket

import numpy as np
import pytest

from gpu_helpers import poison, to_numpy, to_torch

pytestmark = pytest.mark.gpu


def _ring_nvls(R, coll, n, extra=""):
    text = R.rescclGenerateIr("ring", coll, n)
    hdr, rest = (text.split("\n", 1) + [""])[:2]
    return hdr + " nvls=1 " + extra + "\n" + rest


def _alloc_or_skip(R, comms, nbytes):
    try:
        return R.rescclNvlsAllocAll(comms, nbytes)
    except R.ResCCLError as e:
        assert e.code == R.rescclCudaError, str(e)
        assert "cuMulticast" in str(e), str(e)
        pytest.skip(f"multicast refused on this box: {e}")


@pytest.mark.parametrize("coll", ["allreduce", "reducescatter", "allgather"])
@pytest.mark.parametrize("dtype", ["bfloat16", "float32", "int32", "float16"])
def test_nvls_single_rank_window_parity(coll, dtype):
    """N = 1 (the only NVLS group one GPU can form): the multicast object has one device,
    mred is the identity and mcast a copy -- every multimem instruction, barrier and the
    routing still run.  Vector and 4-byte-granule paths, in- and out-of-place."""
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    from paper_conf_sigcomm_liuhlgcwz025_b200.torch_api import Communicator, tensor_at
    from oracle import nvls
    import resccl_inputs as inp
    tdt = {"bfloat16": torch.bfloat16, "float32": torch.float32, "int32": torch.int32,
           "float16": torch.float16}[dtype]
    h = R.rescclCommInitAll([0])
    comm = Communicator(h[0])
    try:
        assert isinstance(R.rescclNvlsSupported(h[0]), bool)
        nbytes = 8 << 20
        (ptr,) = _alloc_or_skip(R, h, nbytes)
        comm.load(_ring_nvls(R, coll, 1))
        e = torch.tensor([], dtype=tdt).element_size()
        win = tensor_at(ptr, nbytes // e, tdt)
        # (count, element offset): 16-byte granules; 16-byte granules + 4-byte tail; tiny;
        # 4-byte granules only; bf16/fp16 ineligible (odd count / 2-byte offset -> the
        # ring plan runs inside the window)
        for count, off in [(1 << 20, 0), (4098, 8), (2, 4096), (262150, 2), (1001, 3)]:
            half = (nbytes // e) // 2
            x = inp.rank_input(dtype, 5, 0, count)
            s = win[off:off + count]
            s.copy_(to_torch(x, dtype))
            r = win[half + off:half + off + count]
            poison(r)
            getattr(comm, coll)(s, r)
            torch.cuda.synchronize()
            assert comm.async_error() == 0
            exp = nvls.replay(coll, [x], dtype)[0]
            assert np.array_equal(to_numpy(r, dtype).view(np.uint8), exp.view(np.uint8)), (count, off)
        R.rescclNvlsFree(h[0], ptr)
    finally:
        comm.destroy()


@pytest.mark.parametrize("coll", ["allreduce", "reducescatter", "allgather"])
def test_nvls_algorithm_falls_back_on_virtual_ranks(coll):
    """Virtual ranks share one device, so nvls=1 never applies: the ring plan runs."""
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    import resccl_inputs as inp
    from gpu_helpers import run_virtual
    from oracle import definition
    n, count, dtype = 4, 5000, "int32"
    xs = [inp.rank_input(dtype, 2, r, count * (n if coll == "reducescatter" else 1)) for r in range(n)]
    out, info, err = run_virtual(R, _ring_nvls(R, coll, n, "chunkbytes=4096"), coll, xs, dtype, count)
    assert err == 0 and info["nvls"] == 1
    ref = {"allreduce": lambda: definition.allreduce(xs, dtype),
           "reducescatter": lambda: definition.reducescatter(xs, dtype),
           "allgather": lambda: definition.allgather(xs)}[coll]()
    for a, b in zip(out, ref):
        assert np.array_equal(a, b)


def test_nvls_algorithm_falls_back_outside_windows():
    """One-device communicator, nvls=1, buffers from torch (not in an NVLS window): the
    primitive plan runs and the result is the definition's."""
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    from paper_conf_sigcomm_liuhlgcwz025_b200.torch_api import Communicator
    import resccl_inputs as inp
    h = R.rescclCommInitAll([0])
    comm = Communicator(h[0])
    try:
        comm.load(_ring_nvls(R, "allreduce", 1))
        x = inp.rank_input("float32", 4, 0, 10001)
        s = to_torch(x, "float32")
        r = torch.empty_like(s)
        poison(r)
        comm.allreduce(s, r)
        torch.cuda.synchronize()
        assert np.array_equal(to_numpy(r, "float32").view(np.uint32), x.view(np.uint32))
    finally:
        comm.destroy()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _alloc_worker(rank, world, port, q):
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        comm = R.init_process_group_comm(rank, world, 0)
        res = None
        try:
            ptr = comm.nvls_alloc(4 << 20)
            res = ("ok", ptr != 0)
            R.rescclNvlsFree(comm.handle, ptr)
        except R.ResCCLError as e:
            res = ("error", e.code, str(e))
        dist.barrier()  # every rank got here: no rank is stuck in the allocation protocol
        comm.destroy()
        dist.destroy_process_group()
        q.put((rank, res, None))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, None, traceback.format_exc()))


@pytest.mark.timeout(240)
def test_nvls_multiprocess_alloc_protocol():
    """Two processes on cuda:0: one device cannot be added to a multicast object twice (and
    the gpurun boxes refuse multicast altogether), so every rank must report the same
    CudaError -- naming the failing rank and call -- and return."""
    import torch.multiprocessing as mp
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_alloc_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, out, tb = q.get(timeout=220)
        assert tb is None, tb
        res[rank] = out
    for p in procs:
        p.join(timeout=60)
    kinds = {res[r][0] for r in range(world)}
    assert len(kinds) == 1, res  # all ranks agree
    if kinds == {"error"}:
        for r in range(world):
            assert res[r][1] == R.rescclCudaError, res[r]
            assert "NVLS window" in res[r][2] and "failed on rank" in res[r][2], res[r]
