"""API rules of include/resccl.h that fix round-1 review findings:

* ReduceScatter scratch may not grow inside a CUDA-graph capture (InvalidUsage), and a
  capture after an eager call of that size works;
* multi-process ranks must agree on RESCCL_HOST_PIECE (rescclCommConnect: InvalidUsage);
* single-process multi-device communicators refuse pageable host buffers (skipped with
  fewer than 2 GPUs)."""
import os
import socket

import numpy as np
import pytest

import resccl_inputs as inp
from oracle import definition

pytestmark = pytest.mark.gpu


def test_reducescatter_scratch_growth_refused_in_capture():
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n, cnt = 4, 5000
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(R.rescclGenerateIr("ring", "reducescatter", n) + "")
        xs = [torch.from_numpy(inp.rank_input("int32", 2, r, n * cnt)).cuda() for r in range(n)]
        ys = [torch.empty(cnt, dtype=torch.int32, device="cuda") for _ in range(n)]
        st = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with pytest.raises(R.ResCCLError) as ei:
            with torch.cuda.graph(g, stream=st):
                grp.reducescatter(xs, ys, stream=st)
        assert ei.value.code == R.rescclInvalidUsage
    finally:
        grp.destroy()
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(R.rescclGenerateIr("ring", "reducescatter", n))
        grp.reducescatter(xs, ys)          # eager call of this size grows the scratch
        torch.cuda.synchronize()
        st = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            grp.reducescatter(xs, ys, stream=st)
        for t in ys:
            t.zero_()
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        exp = definition.reducescatter([inp.rank_input("int32", 2, r, n * cnt) for r in range(n)], "int32")
        for r in range(n):
            assert np.array_equal(ys[r].cpu().numpy(), exp[r])
    finally:
        grp.destroy()


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _piece_worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        os.environ["RESCCL_HOST_PIECE"] = str((8 << 20) * (rank + 1))
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        h = R.rescclCommCreate(rank, world, dev)
        blobs = [None] * world
        dist.all_gather_object(blobs, R.rescclCommGetHandle(h))
        try:
            R.rescclCommConnect(h, blobs)
            res = "connected"
        except R.ResCCLError as e:
            res = (e.code, R.rescclGetLastError())
        R.rescclCommDestroy(h)
        dist.destroy_process_group()
        q.put((rank, res, None))
    except Exception:
        import traceback
        q.put((rank, None, traceback.format_exc()))


@pytest.mark.timeout(200)
def test_host_piece_must_agree_across_processes():
    import torch.multiprocessing as mp
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_piece_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=180) for _ in range(2)]
    for p in ps:
        p.join(20)
    for rank, res, tb in out:
        assert tb is None, tb
        assert res[0] == R.rescclInvalidUsage and "RESCCL_HOST_PIECE" in res[1], res


def test_pageable_refused_single_process_multi_device():
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs")
    grp = R.VirtualGroup(2, devices=[0, 1])
    try:
        s = [torch.ones(1000, dtype=torch.float32) for _ in range(2)]   # pageable host memory
        r = [torch.empty(1000, dtype=torch.float32) for _ in range(2)]
        with pytest.raises(R.ResCCLError) as ei:
            grp.comms[0].allreduce(s[0], r[0])
        assert ei.value.code == R.rescclInvalidArgument
    finally:
        grp.destroy()
