"""f4: PyTorch DDP with its gradient-bucket AllReduce replaced by ResCCL (comm hook).
Two processes on cuda:(rank % device_count) (CUDA IPC; NVLink on a multi-GPU box); the resulting gradients equal the manual average
of both ranks' local gradients."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        from paper_conf_sigcomm_liuhlgcwz025_b200.ddp import ResCCLHookState, resccl_allreduce_hook
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        torch.manual_seed(0)
        model = torch.nn.Sequential(torch.nn.Linear(256, 512), torch.nn.GELU(), torch.nn.Linear(512, 64)).cuda()
        ref = [p.detach().clone() for p in model.parameters()]
        comm = R.init_process_group_comm(rank, world, dev)
        ddp = torch.nn.parallel.DistributedDataParallel(model, device_ids=[dev], bucket_cap_mb=1)
        state = ResCCLHookState(comm)
        ddp.register_comm_hook(state, resccl_allreduce_hook)
        torch.manual_seed(100 + rank)
        x = torch.randn(32, 256, device=f"cuda:{dev}")
        loss = ddp(x).square().mean()
        loss.backward()
        torch.cuda.synchronize()
        grads = [p.grad.detach().cpu().numpy() for p in model.parameters()]
        # local gradients of this rank's batch (no DDP) for the reference average
        m2 = torch.nn.Sequential(torch.nn.Linear(256, 512), torch.nn.GELU(), torch.nn.Linear(512, 64)).cuda()
        with torch.no_grad():
            for a, b in zip(m2.parameters(), ref):
                a.copy_(b)
        m2(x).square().mean().backward()
        local = [p.grad.detach().cpu().numpy() for p in m2.parameters()]
        allocal = [None] * world
        dist.all_gather_object(allocal, local)
        err = comm.async_error()
        dist.barrier()
        comm.destroy()
        dist.destroy_process_group()
        q.put((rank, grads, allocal, state.calls, err, None))
    except Exception:
        import traceback
        q.put((rank, None, None, 0, None, traceback.format_exc()))


@pytest.mark.timeout(300)
def test_ddp_gradients_through_resccl():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    os.environ["RESCCL_TIMEOUT_MS"] = "60000"
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=280) for _ in range(2)]
    for p in ps:
        p.join(30)
    for rank, grads, allocal, calls, err, tb in res:
        assert tb is None, tb
        assert err == 0 and calls >= 1
        for k, g in enumerate(grads):
            want = (allocal[0][k] + allocal[1][k]) / 2
            np.testing.assert_allclose(g, want, rtol=1e-5, atol=1e-6)
