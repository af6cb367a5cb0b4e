"""GPU parity of the lane-engine variants of DESIGN §5.12c (r02): one-sided release /
acquire fences (``splitfence``) and grouped posts of dependency-free pull-sends
(``postgroup``).  Neither changes a value or an order of the plan, so every variant must
equal the oracle's replay of its own plan byte for byte: the full mesh (PAPER Fig. 16 at one
node of 8, port link model: seven pull-sends at the head of each send lane -- the grouped
case) and the ring, register path (small slices) and TMA lane engine (large slices),
out of place and in place."""
import numpy as np
import pytest

import resccl_inputs as inp
from gpu_helpers import run_virtual
from oracle import ir as oir, lower, replay

pytestmark = pytest.mark.gpu


def _expect(g, xs, dtype, count, cb, inst, model):
    pl = lower.lower(g, model, direct=True)
    return replay.replay(pl, xs, dtype, count, chunk_bytes=cb, instances=inst, K=2)


@pytest.mark.timeout(600)
@pytest.mark.parametrize("variant", ["splitfence=1 postgroup=1", "splitfence=0 postgroup=0",
                                     "splitfence=1 postgroup=0", "splitfence=0 postgroup=1"])
@pytest.mark.parametrize("name,kw,model", [("hm", {"g": 8}, "port"), ("ring", {}, "pair")])
@pytest.mark.parametrize("count,dtype", [(3 * 4096 + 77, "bfloat16"), ((2 << 20) + 4099, "int32")])
@pytest.mark.parametrize("inplace", [False, True])
def test_engine_variants_bit_exact(variant, name, kw, model, count, dtype, inplace):
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    g = oir.generate(name, "allreduce", n, **kw)
    cb = 4096 if count < (1 << 20) else 1 << 20
    opts = dict(chunkbytes=cb, instances=2, fifodepth=2, direct=1, linkmodel=model)
    for k, v in opts.items():
        g.extra[k] = str(v)
    text = g.to_text()
    hdr, rest = text.split("\n", 1)
    xs = inp.all_inputs(dtype, 31, n, count)
    outs, info, err = run_virtual(R, hdr + " " + variant + "\n" + rest, "allreduce", xs, dtype, count, inplace=inplace)
    assert err == 0
    exp = _expect(g, xs, dtype, count, cb, 2, model)
    for r in range(n):
        assert np.array_equal(outs[r].view(np.uint8), exp[r].view(np.uint8)), f"rank {r}"


@pytest.mark.timeout(600)
@pytest.mark.parametrize("name,kw,nwarps,inst,cb", [("hm", {"g": 8}, 2, 1, 32 << 20), ("hm", {"g": 8}, 4, 1, 32 << 20),
                                                    ("hm", {"g": 4}, 4, 4, 512 << 10)])
@pytest.mark.parametrize("count", [3 * 4096 + 77, 131072 + 11, (1 << 20) + 4099])
def test_small_cta_geometries_bit_exact(name, kw, nwarps, inst, cb, count):
    """The small-message classes of the size-tuned selection: 64- and 128-thread
    CTAs.  A one-warp lane (nwarps=2) takes the register path even where slices would select
    the TMA engine (which needs combine warps)."""
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    n = 8
    g = oir.generate(name, "allreduce", n, **kw)
    for k, v in dict(chunkbytes=cb, instances=inst, fifodepth=2, direct=1, nwarps=nwarps).items():
        g.extra[k] = str(v)
    xs = inp.all_inputs("bfloat16", 33, n, count)
    outs, info, err = run_virtual(R, g.to_text(), "allreduce", xs, "bfloat16", count)
    assert err == 0 and info["tma"] == (0 if nwarps < 4 else 1)
    exp = _expect(g, xs, "bfloat16", count, cb, inst, "pair")
    for r in range(n):
        assert np.array_equal(outs[r].view(np.uint8), exp[r].view(np.uint8)), f"rank {r}"
