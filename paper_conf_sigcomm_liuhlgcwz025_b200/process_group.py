"""f4 framework integration: ResCCL as a ``torch.distributed`` backend.

The paper integrates ResCCL into Megatron-LM by "relink and rebuild" (PAPER.md
P:L2624-2628): the training framework keeps calling its collective API and ResCCL's
generated kernels run underneath.  In PyTorch the equivalent seam is a process-group
backend:

    import paper_conf_sigcomm_liuhlgcwz025_b200.process_group  # registers "resccl"
    torch.cuda.set_device(local_rank)
    dist.init_process_group("resccl", rank=rank, world_size=world)   # env:// or store
    dist.all_reduce(t)                       # -> rescclAllReduce on the current stream

Every collective below is argument marshalling onto the C ABI (one ``rescclComm_t``
per process group, bootstrapped through the group's c10d store); the arithmetic runs
in the generated sm_100a kernels.  Semantics:

* ops are enqueued on the caller's current CUDA stream (like NCCL with a single
  stream): the returned Work is complete from the stream's point of view, so
  ``wait()`` is a no-op and later work on that stream sees the result;
* all_reduce: SUM / MAX / MIN map to rescclSum / Max / Min; AVG = SUM then a division
  by the group size (a framework-side scale, as DDP does); other ops raise;
* all_gather_into_tensor / reduce_scatter_tensor map 1:1 to rescclAllGather /
  rescclReduceScatter; the list forms go through one flat buffer;
* broadcast is an AllReduce of the root's bits with zeros from every other rank, done
  on an int32 view when the byte size allows it (bit-exact, -0.0 and NaN payloads
  included) and in the tensor's dtype otherwise (x + 0 = x except -0.0 -> +0.0);
* barrier = a 1-element AllReduce followed by a stream synchronisation.
The collective algorithms are the library defaults (built-in ring) unless loaded with
``ResCCLProcessGroup.load(ir_text)``; RESCCL_* environment options apply (resccl.h).
"""
from __future__ import annotations

from typing import List

import torch
import torch.distributed as dist
from torch.futures import Future

import paper_conf_sigcomm_liuhlgcwz025_b200 as _r
from .torch_api import Communicator

BACKEND = "resccl"

_OPS = {dist.ReduceOp.SUM: "sum", dist.ReduceOp.MAX: "max", dist.ReduceOp.MIN: "min"}


def _op_name(op) -> str:
    op = getattr(op, "op", op)  # options carry a ReduceOp object; its .op is the RedOpType
    if op in _OPS:
        return _OPS[op]
    if op == dist.ReduceOp.AVG:
        return "avg"
    raise ValueError(f"ResCCL backend: unsupported reduce op {op}")


def _as_words(t: torch.Tensor) -> torch.Tensor:
    """A dtype-agnostic view for pure data movement (AllGather, Broadcast): 32-bit words
    when the byte count allows, else 16-bit (carried as float16 -- moved, never added)."""
    nbytes = t.numel() * t.element_size()
    if t.dtype in (torch.int32, torch.float32, torch.float16, torch.bfloat16) and nbytes % 4:
        return t
    if nbytes % 4 == 0:
        return t.view(torch.int32) if t.dtype != torch.int32 else t
    if nbytes % 2 == 0:
        return t.view(torch.float16)
    raise ValueError(f"ResCCL backend: {t.dtype} tensor of {nbytes} bytes is not a whole number of 16-bit words")


class _Done(dist._Work):
    """A Work whose collective is already enqueued on the caller's stream."""

    def __init__(self, result, device):
        super().__init__()
        self._fut = Future(devices=[device])
        self._fut.set_result(result)

    def wait(self, timeout=None):
        return True

    def is_completed(self):
        return True

    def is_success(self):
        return True

    def get_future(self):
        return self._fut


class ResCCLProcessGroup(dist.ProcessGroup):
    def __init__(self, store, rank: int, size: int, timeout=None, device: int = None):
        super().__init__(rank, size)
        self.device = torch.cuda.current_device() if device is None else device
        h = _r.rescclCommCreate(rank, size, self.device)
        store.set(f"resccl/conn/{rank}", _r.rescclCommGetHandle(h))
        blobs = [bytes(store.get(f"resccl/conn/{q}")) for q in range(size)]
        _r.rescclCommConnect(h, blobs)
        self.comm = Communicator(h)
        self.calls = 0

    # ------------------------------------------------------------------ helpers
    def getBackendName(self):
        return BACKEND

    def load(self, ir_text: str) -> int:
        """Load an algorithm (IR text or a ResCCLang program) for its collective."""
        return self.comm.load(ir_text)

    def _check(self, t):
        if not (t.is_cuda and t.device.index == self.device):
            raise ValueError(f"ResCCL backend: tensors must live on cuda:{self.device}, got {t.device}")
        if not t.is_contiguous():
            raise ValueError("ResCCL backend: tensors must be contiguous")

    def _stream(self):
        return torch.cuda.current_stream(self.device).cuda_stream

    def _done(self, result):
        self.calls += 1
        return _Done(result, torch.device("cuda", self.device))

    # ------------------------------------------------------------------ collectives
    def allreduce(self, tensors: List[torch.Tensor], opts):
        op = _op_name(opts.reduceOp)
        for t in tensors:
            self._check(t)
            self.comm.allreduce(t, t, "sum" if op == "avg" else op, stream=self._stream())
            if op == "avg":
                t.div_(self.size())
        return self._done(tensors)

    def _allgather_base(self, output: torch.Tensor, input: torch.Tensor, opts=None):
        self._check(output)
        self._check(input)
        self.comm.allgather(_as_words(input), _as_words(output), stream=self._stream())
        return self._done([output])

    def allgather_into_tensor_coalesced(self, outputs, inputs, opts=None):
        for o, i in zip(outputs, inputs):
            self._allgather_base(o, i, opts)
        return self._done(outputs)

    def allgather(self, output_tensors: List[List[torch.Tensor]], input_tensors: List[torch.Tensor], opts=None):
        for outs, inp in zip(output_tensors, input_tensors):
            self._check(inp)
            flat = torch.empty(self.size() * inp.numel(), dtype=inp.dtype, device=inp.device)
            self.comm.allgather(_as_words(inp), _as_words(flat), stream=self._stream())
            for q, o in enumerate(outs):
                o.copy_(flat[q * inp.numel():(q + 1) * inp.numel()].view_as(o))
        return self._done(output_tensors)

    def _reduce_scatter_base(self, output: torch.Tensor, input: torch.Tensor, opts):
        op = _op_name(opts.reduceOp)
        self._check(output)
        self._check(input)
        self.comm.reducescatter(input, output, "sum" if op == "avg" else op, stream=self._stream())
        if op == "avg":
            output.div_(self.size())
        return self._done([output])

    def reduce_scatter_tensor_coalesced(self, outputs, inputs, opts):
        for o, i in zip(outputs, inputs):
            self._reduce_scatter_base(o, i, opts)
        return self._done(outputs)

    def reduce_scatter(self, output_tensors: List[torch.Tensor], input_tensors: List[List[torch.Tensor]], opts):
        for out, ins in zip(output_tensors, input_tensors):
            flat = torch.cat([x.reshape(-1) for x in ins])
            self._check(out)
            tmp = torch.empty_like(out)
            op = _op_name(opts.reduceOp)
            self.comm.reducescatter(flat, tmp, "sum" if op == "avg" else op, stream=self._stream())
            if op == "avg":
                tmp.div_(self.size())
            out.copy_(tmp)
        return self._done(output_tensors)

    def broadcast(self, tensors: List[torch.Tensor], opts):
        root = opts.rootRank
        for t in tensors:
            self._check(t)
            if self.rank() != root:
                t.zero_()
            nbytes = t.numel() * t.element_size()
            if nbytes % 4 == 0:
                v = _as_words(t)          # integer sum of the root's words and zeros: bit-exact
            elif t.dtype in (torch.float16, torch.bfloat16):
                v = t                     # x + 0 = x except -0.0 -> +0.0
            else:
                raise ValueError(f"ResCCL backend: broadcast of {t.dtype} with {nbytes} bytes is unsupported")
            if v.numel():
                self.comm.allreduce(v, v, "sum", stream=self._stream())
        return self._done(tensors)

    def barrier(self, opts=None):
        t = torch.zeros(1, dtype=torch.int32, device=f"cuda:{self.device}")
        self.comm.allreduce(t, t, "sum", stream=self._stream())
        torch.cuda.current_stream(self.device).synchronize()
        return self._done([t])

    def shutdown(self):
        self.comm.destroy()


def _create(store, rank, size, timeout):
    return ResCCLProcessGroup(store, rank, size, timeout)


def register() -> None:
    if BACKEND not in dist.Backend.backend_list:
        dist.Backend.register_backend(BACKEND, _create, devices=["cuda"])


register()
