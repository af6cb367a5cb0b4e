"""Thin tensor-level helpers over the C ABI (argument marshalling only).

``Communicator`` wraps one rank's ``rescclComm_t``; ``VirtualGroup`` wraps the
single-process virtual ranks of one GPU (``rescclCommInitAll`` with a repeated
device).  ``init_process_group_comm`` bootstraps a multi-process communicator by
exchanging the connection blobs with ``torch.distributed.all_gather_object``.
"""
from __future__ import annotations

from typing import List, Optional, Sequence

import paper_conf_sigcomm_liuhlgcwz025_b200 as _r

_TORCH_DT = {"torch.int32": _r.rescclInt32, "torch.float32": _r.rescclFloat32,
             "torch.float16": _r.rescclFloat16, "torch.bfloat16": _r.rescclBfloat16}


def dtype_of(t) -> int:
    d = _TORCH_DT.get(str(t.dtype))
    if d is None:
        raise TypeError(f"unsupported dtype {t.dtype}")
    return d


def _stream(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return stream if isinstance(stream, int) else stream.cuda_stream


class Communicator:
    def __init__(self, handle: int):
        self.handle = handle
        self.rank = _r.rescclCommRank(handle)
        self.nranks = _r.rescclCommCount(handle)
        self.algos = []

    def load(self, ir_text: str) -> int:
        a = _r.rescclLoadAlgorithm(self.handle, ir_text)
        self.algos.append(a)
        return a

    def allreduce(self, send, recv, op: str = "sum", stream=None):
        # device tensors, or host tensors (pinned for async copies): the library stages
        # host buffers through device memory itself (include/resccl.h, host buffers)
        assert send.numel() == recv.numel()
        _r.rescclAllReduce(send.data_ptr(), recv.data_ptr(), send.numel(), dtype_of(send), _r.OPS[op],
                           self.handle, _stream(stream))

    def allgather(self, send, recv, stream=None):
        assert recv.numel() == send.numel() * self.nranks
        _r.rescclAllGather(send.data_ptr(), recv.data_ptr(), send.numel(), dtype_of(send), self.handle,
                           _stream(stream))

    def reducescatter(self, send, recv, op: str = "sum", stream=None):
        assert send.numel() == recv.numel() * self.nranks
        _r.rescclReduceScatter(send.data_ptr(), recv.data_ptr(), recv.numel(), dtype_of(send), _r.OPS[op],
                               self.handle, _stream(stream))

    def async_error(self) -> int:
        return _r.rescclCommGetAsyncError(self.handle)

    def register(self, tensor, group=None) -> int:
        """Register `tensor` as a symmetric window (collective over the process group):
        export, exchange the blobs with all_gather_object, map the peers' windows."""
        import torch.distributed as dist
        blob = _r.rescclCommRegister(self.handle, tensor.data_ptr(), tensor.numel() * tensor.element_size())
        blobs: List[Optional[bytes]] = [None] * self.nranks
        dist.all_gather_object(blobs, blob, group=group)
        return _r.rescclCommRegisterConnect(self.handle, blobs)

    def nvls_alloc(self, nbytes: int, group=None) -> int:
        """Allocate an NVLS window (f3; collective over the process group): the fabric
        handle and status rounds travel through all_gather_object."""
        import torch.distributed as dist

        def ag(blob: bytes):
            out: List[Optional[bytes]] = [None] * self.nranks
            dist.all_gather_object(out, blob, group=group)
            return out
        return _r.rescclNvlsAlloc(self.handle, nbytes, ag)

    def destroy(self):
        if self.handle:
            _r.rescclCommDestroy(self.handle)
            self.handle = 0


class VirtualGroup:
    """N virtual ranks on one GPU; every collective is issued for all ranks and runs
    as one kernel (see resccl.h, "Execution modes").  With ``devices`` (distinct GPUs,
    one rank each) the same object drives the single-process multi-device mode: one
    kernel per rank over peer memory (cudaDeviceEnablePeerAccess, NVLink)."""

    def __init__(self, nranks: int, device: int = 0, devices: Optional[Sequence[int]] = None):
        devs = list(devices) if devices is not None else [device] * nranks
        assert len(devs) == nranks
        self.comms = [Communicator(h) for h in _r.rescclCommInitAll(devs)]
        self.nranks = nranks
        self.devices = devs

    def load(self, ir_text: str) -> List[int]:
        return [c.load(ir_text) for c in self.comms]

    def plan_info(self) -> dict:
        return _r.rescclGetPlanInfo(self.comms[0].algos[-1])

    def allreduce(self, sends: Sequence, recvs: Sequence, op: str = "sum", stream=None):
        for c, s, r in zip(self.comms, sends, recvs):
            c.allreduce(s, r, op, stream)

    def allgather(self, sends, recvs, stream=None):
        for c, s, r in zip(self.comms, sends, recvs):
            c.allgather(s, r, stream)

    def reducescatter(self, sends, recvs, op: str = "sum", stream=None):
        for c, s, r in zip(self.comms, sends, recvs):
            c.reducescatter(s, r, op, stream)

    def async_error(self) -> int:
        return self.comms[0].async_error()

    def destroy(self):
        for c in self.comms:
            c.destroy()


class _CudaArray:
    """__cuda_array_interface__ over a raw device pointer (an NVLS window)."""

    def __init__(self, ptr: int, shape, typestr: str):
        self.__cuda_array_interface__ = {"data": (ptr, False), "shape": tuple(shape), "typestr": typestr,
                                         "version": 3, "strides": None}


def tensor_at(ptr: int, numel: int, dtype, device: int = 0):
    """A torch tensor viewing `numel` elements at device pointer `ptr` (not owning it):
    how NVLS windows are handed to torch.  bf16 has no typestr, so it is viewed via int16."""
    import torch
    ts = {torch.float32: "<f4", torch.float16: "<f2", torch.int32: "<i4", torch.bfloat16: "<i2"}[dtype]
    with torch.cuda.device(device):
        t = torch.as_tensor(_CudaArray(ptr, (numel,), ts), device=f"cuda:{device}")
    return t.view(torch.bfloat16) if dtype == torch.bfloat16 else t


def init_process_group_comm(rank: int, nranks: int, device: int, group=None) -> Communicator:
    """Multi-process bootstrap: Create -> GetHandle -> all_gather_object -> Connect."""
    import torch.distributed as dist
    h = _r.rescclCommCreate(rank, nranks, device)
    blob = _r.rescclCommGetHandle(h)
    blobs: List[Optional[bytes]] = [None] * nranks
    dist.all_gather_object(blobs, blob, group=group)
    _r.rescclCommConnect(h, blobs)
    return Communicator(h)
