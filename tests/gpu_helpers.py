"""Shared helpers of the GPU parity tests: run a collective through the C ABI on
virtual ranks of cuda:0 and produce the oracle's expectation for the same inputs."""
from __future__ import annotations

import numpy as np

import resccl_inputs as inp
from oracle import definition, ir as oir, lower, replay

TORCH_DT = {"int32": "int32", "float32": "float32", "float16": "float16", "bfloat16": "bfloat16"}


def to_torch(x: np.ndarray, dtype: str, device="cuda:0"):
    """device "cuda:0", "pinned" (page-locked host) or "cpu" (pageable host)."""
    import torch
    if dtype == "bfloat16":
        t = torch.from_numpy(x.view(np.int16).copy()).view(torch.bfloat16)
    else:
        t = torch.from_numpy(x.copy())
    if device == "pinned":
        return t.pin_memory()
    return t.to(device)


def to_numpy(t, dtype: str) -> np.ndarray:
    import torch
    t = t.cpu()
    if dtype == "bfloat16":
        return t.view(torch.int16).numpy().view(np.uint16).copy()
    return t.numpy().copy()


def poison(t):
    import torch
    if t.dtype in (torch.float32, torch.float16, torch.bfloat16):
        t.fill_(float("nan"))
    else:
        t.fill_(0x5A5A5A5A)


def run_virtual(R, ir_text: str, coll: str, xs, dtype: str, count: int, op: str = "sum",
                inplace: bool = False, iters: int = 1, send_dev: str = "cuda:0", recv_dev: str = "cuda:0"):
    """Load ``ir_text`` on len(xs) virtual ranks of cuda:0, run ``iters`` times, return
    (outputs as numpy, plan info, async error).  send_dev / recv_dev: where the buffers
    live ("cuda:0", "pinned" or "cpu" host memory; in-place uses send_dev for both)."""
    import torch
    n = len(xs)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(ir_text)
        info = grp.plan_info()
        sends = [to_torch(x, dtype, send_dev) for x in xs]

        def empty(m, like):
            if send_dev in ("pinned", "cpu") and inplace or recv_dev in ("pinned", "cpu") and not inplace:
                t = torch.empty(m, dtype=like.dtype)
                return t.pin_memory() if (send_dev if inplace else recv_dev) == "pinned" else t
            return torch.empty(m, dtype=like.dtype, device="cuda:0")
        recvs = []
        for r in range(n):
            if inplace:
                if coll == "allreduce":
                    recvs.append(sends[r])
                elif coll == "allgather":
                    big = empty(n * count, sends[r])
                    poison(big)
                    big[r * count:(r + 1) * count].copy_(sends[r])
                    sends[r] = big[r * count:(r + 1) * count]
                    recvs.append(big)
                else:
                    recvs.append(sends[r][r * count:(r + 1) * count])
            else:
                m = count * n if coll == "allgather" else count
                t = empty(m, sends[r])
                poison(t)
                recvs.append(t)
        for _ in range(iters):
            if inplace and iters > 1:
                raise ValueError("in-place runs are single-shot")
            getattr(grp, coll)(sends, recvs, op) if coll != "allgather" else grp.allgather(sends, recvs)
        torch.cuda.synchronize()
        err = grp.async_error()
        outs = [to_numpy(t, dtype) for t in recvs]
        return outs, info, err
    finally:
        grp.destroy()


def oracle_expect(g, xs, dtype, count, op="sum", chunk_bytes=1 << 20, instances=1, K=4, model="pair"):
    pl = lower.lower(g, model)
    return replay.replay(pl, xs, dtype, count, op=op, chunk_bytes=chunk_bytes, instances=instances, K=K)


def definition_expect(coll, xs, dtype, op="sum"):
    if coll == "allreduce":
        return definition.allreduce(xs, dtype, op)
    if coll == "allgather":
        return definition.allgather(xs)
    return definition.reducescatter(xs, dtype, op)
