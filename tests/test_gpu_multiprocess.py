"""Multi-process path (one process per rank, CUDA-IPC-mapped peer arenas, .sys-scope
flags).  Rank r runs on cuda:(r % device_count): on a one-GPU box every process shares
cuda:0 (CUDA IPC works between processes of one device); on a multi-GPU box the same
tests cross NVLink.  Results are compared with the oracle."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, algo, coll, count, dtype, q, opts="chunkbytes=4096 instances=2 fifodepth=2",
            where="cuda:0"):
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        sys.path.insert(0, os.path.join(root, "tests"))
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        import resccl_inputs as inp
        from gpu_helpers import to_numpy, to_torch, poison
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = R.init_process_group_comm(rank, world, dev)
        text = R.rescclGenerateIr(algo, coll, world)
        hdr, rest = text.split("\n", 1)
        comm.load(hdr + " " + opts + "\n" + rest)
        m = count * world if coll == "reducescatter" else count
        x = inp.rank_input(dtype, 3, rank, m)
        s = to_torch(x, dtype, f"cuda:{dev}" if where.startswith("cuda") else where)
        outs = []
        for it in range(2):  # two calls: monotone flags across calls
            n_out = count * world if coll == "allgather" else count
            r = torch.empty(n_out, dtype=s.dtype, device="cpu" if where == "pinned" else f"cuda:{dev}")
            if where == "pinned":
                r = r.pin_memory()
            poison(r)
            getattr(comm, coll)(s, r)
            torch.cuda.synchronize()
            outs.append(to_numpy(r, dtype))
        err = comm.async_error()
        dist.barrier()
        comm.destroy()
        dist.destroy_process_group()
        q.put((rank, outs, err, None))
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, None, None, traceback.format_exc()))


@pytest.mark.timeout(240)
@pytest.mark.parametrize("algo,coll,world,where", [("ring", "allreduce", 2, "cuda:0"), ("ring", "allgather", 2, "cuda:0"),
                                                   ("ring", "reducescatter", 2, "cuda:0"), ("dbt", "allreduce", 4, "cuda:0"),
                                                   ("ring", "allreduce", 2, "pinned"), ("ring", "allgather", 2, "pinned"),
                                                   ("ring", "reducescatter", 2, "pinned")])
def test_ipc_processes_match_oracle(algo, coll, world, where):
    """where = "pinned": host send/receive buffers, staged by the library (host_rank)."""
    import torch.multiprocessing as mp
    import resccl_inputs as inp
    from oracle import ir as oir, lower, replay
    count, dtype = 9000, "float32"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    env_old = os.environ.get("RESCCL_TIMEOUT_MS")
    os.environ["RESCCL_TIMEOUT_MS"] = "60000"
    procs = [ctx.Process(target=_worker, args=(r, world, port, algo, coll, count, dtype, q),
                         kwargs={"where": where}) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, outs, err, tb = q.get(timeout=220)
        assert tb is None, tb
        res[rank] = (outs, err)
    for p in procs:
        p.join(30)
    if env_old is None:
        os.environ.pop("RESCCL_TIMEOUT_MS", None)
    g = oir.generate(algo, coll, world)
    m = count * world if coll == "reducescatter" else count
    xs = [inp.rank_input(dtype, 3, r, m) for r in range(world)]
    exp = replay.replay(lower.lower(g), xs, dtype, count, chunk_bytes=4096, instances=2, K=2)
    for r in range(world):
        outs, err = res[r]
        assert err == 0
        for o in outs:
            assert np.array_equal(o.view(np.uint8), exp[r].view(np.uint8)), f"rank {r}"


@pytest.mark.timeout(300)
@pytest.mark.parametrize("algo,coll,world", [("ring", "allreduce", 2), ("ring", "allgather", 2)])
def test_ipc_tma_engine_matches_oracle(algo, coll, world):
    """Slices above tmamin: the TMA lane engine with .sys-scope flags across processes."""
    import torch.multiprocessing as mp
    import resccl_inputs as inp
    from oracle import ir as oir, lower, replay
    count, dtype = (6 << 20) + 33, "float32"
    opts = "chunkbytes=4194304 instances=2 fifodepth=2"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    os.environ["RESCCL_TIMEOUT_MS"] = "120000"
    procs = [ctx.Process(target=_worker, args=(r, world, port, algo, coll, count, dtype, q, opts))
             for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, outs, err, tb = q.get(timeout=280)
        assert tb is None, tb
        res[rank] = (outs, err)
    for p in procs:
        p.join(30)
    g = oir.generate(algo, coll, world)
    m = count * world if coll == "reducescatter" else count
    xs = [inp.rank_input(dtype, 3, r, m) for r in range(world)]
    exp = replay.replay(lower.lower(g), xs, dtype, count, chunk_bytes=4194304, instances=2, K=2)
    for r in range(world):
        outs, err = res[r]
        assert err == 0
        for o in outs:
            assert np.array_equal(o.view(np.uint8), exp[r].view(np.uint8)), f"rank {r}"


def _window_worker(rank, world, port, algo, coll, count, dtype, q, opts):
    """Direct transport across processes: buffers registered as symmetric windows run
    the direct kernel; an unregistered buffer runs the staged twin (reading R23)."""
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        sys.path.insert(0, os.path.join(root, "tests"))
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        import resccl_inputs as inp
        from gpu_helpers import to_numpy, to_torch, poison
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = R.init_process_group_comm(rank, world, dev)
        text = R.rescclGenerateIr(algo, coll, world)
        hdr, rest = text.split("\n", 1)
        comm.load(hdr + " " + opts + "\n" + rest)
        m = count * world if coll == "reducescatter" else count
        n_out = count * world if coll == "allgather" else count
        x = to_torch(inp.rank_input(dtype, 3, rank, m), dtype, f"cuda:{dev}")
        # one window holding send and receive buffers at symmetric offsets
        win = torch.empty(m + n_out + 64, dtype=x.dtype, device=f"cuda:{dev}")
        comm.register(win)
        s_reg, r_reg = win[:m], win[m + 64:m + 64 + n_out]
        s_reg.copy_(x)
        outs = []
        for it, reg in enumerate([True, False, True, True]):
            s = s_reg if reg else x
            r = r_reg if reg else torch.empty(n_out, dtype=x.dtype, device=f"cuda:{dev}")
            poison(r)
            torch.cuda.synchronize()
            dist.barrier()
            getattr(comm, coll)(s, r)
            torch.cuda.synchronize()
            outs.append(to_numpy(r.clone(), dtype))
        err = comm.async_error()
        dist.barrier()
        comm.destroy()
        dist.destroy_process_group()
        q.put((rank, outs, err, None))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, None, None, traceback.format_exc()))


@pytest.mark.timeout(300)
@pytest.mark.parametrize("algo,coll,world,count,opts", [
    ("ring", "allreduce", 2, 9000, "chunkbytes=4096 instances=2 fifodepth=2 direct=1"),
    ("ring", "allgather", 2, 9000, "chunkbytes=4096 instances=2 fifodepth=2 direct=1"),
    ("ring", "reducescatter", 2, 9000, "chunkbytes=4096 instances=2 fifodepth=2 direct=1"),
    ("dbt", "allreduce", 4, 9000, "chunkbytes=4096 instances=2 fifodepth=2 direct=1"),
    ("ring", "allreduce", 2, (6 << 20) + 33, "chunkbytes=4194304 instances=2 fifodepth=2 direct=1"),
    # push-reduce (R31): rrc operands pushed into the receiver's FIFO, recv payloads pushed directly
    ("ring", "allreduce", 2, 9000, "chunkbytes=4096 instances=2 fifodepth=2 direct=1 pushreduce=1"),
    ("dbt", "allreduce", 4, 9000, "chunkbytes=4096 instances=2 fifodepth=2 direct=1 pushreduce=1"),
    ("ring", "allreduce", 2, (6 << 20) + 33, "chunkbytes=4194304 instances=2 fifodepth=2 direct=1 pushreduce=1"),
])
def test_ipc_registered_windows_direct(algo, coll, world, count, opts):
    import torch.multiprocessing as mp
    import resccl_inputs as inp
    from oracle import ir as oir, lower, replay
    dtype = "float32"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    os.environ["RESCCL_TIMEOUT_MS"] = "120000"
    procs = [ctx.Process(target=_window_worker, args=(r, world, port, algo, coll, count, dtype, q, opts))
             for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, outs, err, tb = q.get(timeout=280)
        assert tb is None, tb
        res[rank] = (outs, err)
    for p in procs:
        p.join(30)
    g = oir.generate(algo, coll, world)
    m = count * world if coll == "reducescatter" else count
    xs = [inp.rank_input(dtype, 3, r, m) for r in range(world)]
    cb = int(opts.split("chunkbytes=")[1].split()[0])
    exp_d = replay.replay(lower.lower(g, direct=True), xs, dtype, count, chunk_bytes=cb, instances=2, K=2)
    exp_s = replay.replay(lower.lower(g), xs, dtype, count, chunk_bytes=cb, instances=2, K=2)
    for r in range(world):
        outs, err = res[r]
        assert err == 0
        for it, o in enumerate(outs):
            e = exp_s if (it == 1 or coll == "reducescatter") else exp_d
            assert np.array_equal(o.view(np.uint8), e[r].view(np.uint8)), f"rank {r} call {it}"


def _graph_worker(rank, world, port, count, q):
    """Device-side epochs across processes: a CUDA graph of a registered-window (direct,
    exit barrier) AllReduce and an unregistered (staged twin) one, replayed between eager
    calls of both plans."""
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        sys.path.insert(0, os.path.join(root, "tests"))
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        import resccl_inputs as inp
        from gpu_helpers import to_numpy, to_torch
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = R.init_process_group_comm(rank, world, dev)
        text = R.rescclGenerateIr("ring", "allreduce", world)
        hdr, rest = text.split("\n", 1)
        comm.load(hdr + " chunkbytes=65536 instances=2 fifodepth=2 direct=1\n" + rest)
        x = to_torch(inp.rank_input("int32", 9, rank, count), "int32", f"cuda:{dev}")
        win = torch.zeros(2 * count + 64, dtype=torch.int32, device=f"cuda:{dev}")
        comm.register(win)
        s_reg, r_reg = win[:count], win[count + 64:2 * count + 64]
        s_reg.copy_(x)
        r_un = torch.zeros(count, dtype=torch.int32, device=f"cuda:{dev}")
        comm.allreduce(s_reg, r_reg)  # eager warm-up: both plans compiled outside the capture
        comm.allreduce(x, r_un)
        torch.cuda.synchronize()
        dist.barrier()
        st = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            comm.allreduce(s_reg, r_reg, stream=st)
            comm.allreduce(x, r_un, stream=st)
        outs = []
        for it in range(3):
            r_reg.zero_()
            r_un.zero_()
            torch.cuda.synchronize()
            dist.barrier()
            g.replay()
            torch.cuda.synchronize()
            outs.append((to_numpy(r_reg.clone(), "int32"), to_numpy(r_un.clone(), "int32")))
            dist.barrier()
            comm.allreduce(s_reg, r_reg)  # eager calls advance the same device epochs
            comm.allreduce(x, r_un)
            torch.cuda.synchronize()
            outs.append((to_numpy(r_reg.clone(), "int32"), to_numpy(r_un.clone(), "int32")))
        err = comm.async_error()
        dist.barrier()
        comm.destroy()
        dist.destroy_process_group()
        q.put((rank, outs, err, None))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, None, None, traceback.format_exc()))


@pytest.mark.timeout(300)
def test_ipc_cuda_graph_replay_device_epochs():
    import torch.multiprocessing as mp
    import resccl_inputs as inp
    from oracle import definition
    world, count = 2, 50000 + 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    os.environ["RESCCL_TIMEOUT_MS"] = "120000"
    procs = [ctx.Process(target=_graph_worker, args=(r, world, port, count, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, outs, err, tb = q.get(timeout=280)
        assert tb is None, tb
        res[rank] = (outs, err)
    for p in procs:
        p.join(30)
    xs = [inp.rank_input("int32", 9, r, count) for r in range(world)]
    exp = definition.allreduce(xs, "int32")
    for r in range(world):
        outs, err = res[r]
        assert err == 0
        for k, (a, b) in enumerate(outs):
            assert np.array_equal(a, exp[r]), f"rank {r} step {k} (window)"
            assert np.array_equal(b, exp[r]), f"rank {r} step {k} (twin)"
