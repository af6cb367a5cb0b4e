"""N>1 host-side logic on CPU (gloo, world_size 2): every rank builds the identical plan
and kernel source from the same IR (the paper's offline compiler is deterministic,
P:L2339-2359), the connection-blob exchange round-trips through
torch.distributed.all_gather_object, and bench.py's max-over-ranks timing works."""
import os
import socket

import pytest


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import torch.distributed as dist
        import paper_conf_sigcomm_liuhlgcwz025_b200 as R
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        text = R.rescclGenerateIr("hm", "allreduce", 8, "g=4")
        plan = R.rescclPlanIr(text, "instances=2")
        src = R.rescclCodegenIr(text, "instances=2", rank, rank + 1)
        objs = [None] * world
        dist.all_gather_object(objs, (plan, len(src), bytes([rank]) * 64))
        t = torch.tensor([float(rank + 1)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.destroy_process_group()
        q.put((rank, objs, float(t.item()), None))
    except Exception:
        import traceback
        q.put((rank, None, None, traceback.format_exc()))


@pytest.mark.timeout(120)
def test_gloo_world2_identical_plans_and_exchange():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=100) for _ in range(2)]
    for p in ps:
        p.join(20)
    for rank, objs, mx, tb in out:
        assert tb is None, tb
        assert objs[0][0] == objs[1][0]           # identical plans on both ranks
        assert objs[0][2] == bytes([0]) * 64 and objs[1][2] == bytes([1]) * 64
        assert mx == 2.0
