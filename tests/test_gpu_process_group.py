"""f4: ResCCL as a torch.distributed backend (``dist.init_process_group("resccl")``).

Two processes (rank r on cuda:(r % device_count)), bootstrapped through the c10d store;
every collective of the framework API is checked against the oracle: int32 against the
definitions (bit-exact), fp32 against the replay of the built-in ring (bit-exact), plus
a DDP training step whose gradients equal the manual average of the ranks' gradients."""
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
        import paper_conf_sigcomm_liuhlgcwz025_b200.process_group as pgm
        import resccl_inputs as inp
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group(pgm.BACKEND, rank=rank, world_size=world)
        assert dist.get_backend() == "resccl"
        out = {}
        cnt = 10001
        x = torch.from_numpy(inp.rank_input("int32", 5, rank, cnt, mode="wrap")).cuda()
        t = x.clone()
        dist.all_reduce(t)
        out["ar_sum"] = t.cpu().numpy()
        t = x.clone()
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        out["ar_max"] = t.cpu().numpy()
        f = torch.from_numpy(inp.rank_input("float32", 6, rank, cnt)).cuda()
        t = f.clone()
        dist.all_reduce(t)
        out["ar_f32"] = t.cpu().numpy()
        t = f.clone()
        w = dist.all_reduce(t, op=dist.ReduceOp.AVG, async_op=True)
        w.wait()
        out["ar_avg"] = t.cpu().numpy()
        ag = torch.empty(world * cnt, dtype=torch.int32, device="cuda")
        dist.all_gather_into_tensor(ag, x)
        out["ag"] = ag.cpu().numpy()
        lst = [torch.empty(cnt, dtype=torch.int32, device="cuda") for _ in range(world)]
        dist.all_gather(lst, x)
        out["ag_list"] = np.concatenate([v.cpu().numpy() for v in lst])
        big = torch.from_numpy(inp.rank_input("int32", 7, rank, world * cnt, mode="wrap")).cuda()
        rs = torch.empty(cnt, dtype=torch.int32, device="cuda")
        dist.reduce_scatter_tensor(rs, big)
        out["rs"] = rs.cpu().numpy()
        b = torch.full((cnt,), float(rank) - 0.0, device="cuda")
        if rank == 1:
            b[0] = -0.0
            b[1] = float("nan")
        dist.broadcast(b, src=1)
        out["bc"] = b.cpu().numpy().view(np.uint32)
        dist.barrier()
        # DDP step through the backend (parameter broadcast + gradient buckets)
        torch.manual_seed(0)
        model = torch.nn.Sequential(torch.nn.Linear(64, 128), torch.nn.GELU(), torch.nn.Linear(128, 8)).cuda()
        ref = [p.detach().clone() for p in model.parameters()]
        ddp = torch.nn.parallel.DistributedDataParallel(model, device_ids=[dev], bucket_cap_mb=1)
        torch.manual_seed(100 + rank)
        xb = torch.randn(16, 64, device="cuda")
        ddp(xb).square().mean().backward()
        torch.cuda.synchronize()
        out["grads"] = [p.grad.detach().cpu().numpy() for p in model.parameters()]
        m2 = torch.nn.Sequential(torch.nn.Linear(64, 128), torch.nn.GELU(), torch.nn.Linear(128, 8)).cuda()
        with torch.no_grad():
            for a, r_ in zip(m2.parameters(), ref):
                a.copy_(r_)
        m2(xb).square().mean().backward()
        out["local"] = [p.grad.detach().cpu().numpy() for p in m2.parameters()]
        dist.destroy_process_group()
        q.put((rank, out, None))
    except Exception:
        import traceback
        q.put((rank, None, traceback.format_exc()))


@pytest.mark.timeout(300)
def test_resccl_backend_collectives_and_ddp():
    import torch.multiprocessing as mp
    import resccl_inputs as inp
    from oracle import definition, ir as oir, lower, replay
    world, cnt = 2, 10001
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    os.environ["RESCCL_TIMEOUT_MS"] = "60000"
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = {}
    for _ in range(world):
        rank, out, tb = q.get(timeout=280)
        assert tb is None, tb
        res[rank] = out
    for p in ps:
        p.join(30)
    xs = [inp.rank_input("int32", 5, r, cnt, mode="wrap") for r in range(world)]
    fs = [inp.rank_input("float32", 6, r, cnt) for r in range(world)]
    bigs = [inp.rank_input("int32", 7, r, world * cnt, mode="wrap") for r in range(world)]
    ar = definition.allreduce(xs, "int32")
    mx = definition.allreduce(xs, "int32", "max")
    f32 = replay.replay(lower.lower(oir.ring_allreduce(world)), fs, "float32", cnt)
    ag = definition.allgather(xs)
    rs = definition.reducescatter(bigs, "int32")
    bc = np.full(cnt, 1.0, np.float32).view(np.uint32).copy()
    bc[0] = np.array([-0.0], np.float32).view(np.uint32)[0]
    for r in range(world):
        o = res[r]
        assert np.array_equal(o["ar_sum"], ar[r])
        assert np.array_equal(o["ar_max"], mx[r])
        assert np.array_equal(o["ar_f32"].view(np.uint32), f32[r].view(np.uint32))
        assert np.array_equal(o["ar_avg"], (f32[r] / np.float32(world)).astype(np.float32))
        assert np.array_equal(o["ag"], ag[r]) and np.array_equal(o["ag_list"], ag[r])
        assert np.array_equal(o["rs"], rs[r])
        assert np.array_equal(o["bc"][2:], bc[2:]) and o["bc"][0] == bc[0]
        assert np.isnan(o["bc"][1:2].view(np.float32)[0])
        for g, l0, l1 in zip(o["grads"], res[0]["local"], res[1]["local"]):
            np.testing.assert_allclose(g, (l0 + l1) / 2, rtol=1e-5, atol=1e-6)
