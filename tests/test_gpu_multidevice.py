"""Single-process distinct-device mode (``rescclCommInitAll([0, 1, ...])``: one rank per
GPU, peer access, one kernel per rank over NVLink peer memory).  Skipped on boxes with
fewer than two GPUs; on a multi-GPU box every result must equal the oracle's replay of
the same plan byte for byte (north_star: bit-exact against the schedule's order)."""
import numpy as np
import pytest

import resccl_inputs as inp
from gpu_helpers import oracle_expect, poison, to_numpy, to_torch
from oracle import ir as oir

pytestmark = pytest.mark.gpu


def _ndev():
    import torch
    return torch.cuda.device_count()


@pytest.mark.timeout(300)
@pytest.mark.parametrize("name,coll,n,dtype", [
    ("ring", "allreduce", 2, "float32"), ("ring", "allgather", 2, "bfloat16"),
    ("ring", "reducescatter", 2, "float16"), ("ring", "allreduce", 4, "bfloat16"),
    ("dbt", "allreduce", 4, "float32"), ("ring", "allreduce", 8, "bfloat16"),
    ("hm", "allreduce", 8, "float32"), ("dbt", "allreduce", 8, "int32"),
])
def test_distinct_devices_match_oracle(name, coll, n, dtype):
    if _ndev() < n:
        pytest.skip(f"needs {n} GPUs, this box has {_ndev()}")
    import torch
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    count = 40000 + 3
    g = oir.generate(name, coll, n, **({"g": 4} if name == "hm" else {}))
    g.extra.update({"chunkbytes": "16384", "instances": "2", "fifodepth": "2"})
    m = count * n if coll == "reducescatter" else count
    xs = [inp.rank_input(dtype, 5, r, m) for r in range(n)]
    grp = R.VirtualGroup(n, devices=list(range(n)))
    try:
        grp.load(g.to_text())
        sends = [to_torch(xs[r], dtype, f"cuda:{r}") for r in range(n)]
        n_out = count * n if coll == "allgather" else count
        recvs = []
        for r in range(n):
            t = torch.empty(n_out, dtype=sends[r].dtype, device=f"cuda:{r}")
            poison(t)
            recvs.append(t)
        for _ in range(2):  # monotone flags across calls
            getattr(grp, coll)(sends, recvs) if coll == "allgather" else getattr(grp, coll)(sends, recvs, "sum")
        for r in range(n):
            torch.cuda.synchronize(r)
        assert grp.async_error() == 0
        outs = [to_numpy(t, dtype) for t in recvs]
    finally:
        grp.destroy()
    exp = oracle_expect(g, xs, dtype, count, chunk_bytes=16384, instances=2, K=2)
    for r in range(n):
        assert np.array_equal(outs[r].view(np.uint8), exp[r].view(np.uint8)), f"rank {r}"
