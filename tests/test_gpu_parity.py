"""GPU parity: the CUDA path (C ABI -> generated sm_100a kernels) vs the CPU oracle.

Bit-exact against the oracle's schedule replay for every dtype (reading R8 makes
16-bit results exact too), and within the north_star tolerance against the naive
definition.  Virtual ranks of cuda:0 execute the same generated kernels as the
multi-GPU path (one launch holds every rank's CTAs)."""
import numpy as np
import pytest

import resccl_inputs as inp
from oracle import definition, ir as oir, lower, numerics, replay

from gpu_helpers import definition_expect, oracle_expect, run_virtual

pytestmark = pytest.mark.gpu

R = None


@pytest.fixture(scope="module", autouse=True)
def _lib():
    global R
    import paper_conf_sigcomm_liuhlgcwz025_b200 as mod
    R = mod


def _hdr(g, **kw):
    for k, v in kw.items():
        g.extra[k] = str(v)
    return g.to_text()


def _check_bytes(outs, exp, coll, n, count):
    for r in range(n):
        a, b = outs[r], exp[r]
        assert a.shape == b.shape, (r, a.shape, b.shape)
        if not np.array_equal(a.view(np.uint8), b.view(np.uint8)):
            bad = np.nonzero(a.view(np.uint8) != b.view(np.uint8))[0]
            raise AssertionError(f"rank {r}: {bad.size} bytes differ, first at byte {bad[0]}: "
                                 f"gpu {a[bad[0] // a.itemsize]} oracle {b[bad[0] // b.itemsize]}")


def test_config1_ring_allreduce_4096_fp32_2ranks():
    """BASELINE configs[0]: ring AR of 4096 fp32, 2 ranks, 1 TB, 4 chunks (2 algorithm
    chunks x 2 micro-batches of 1024 elements, reading R7)."""
    g = oir.ring_allreduce(2)
    text = _hdr(g, chunkbytes=4096, instances=1)
    xs = inp.all_inputs("float32", 0, 2, 4096)
    outs, info, err = run_virtual(R, text, "allreduce", xs, "float32", 4096)
    assert err == 0
    assert info["ctas"] == [1, 1] and info["blocks_per_rank"] == [1, 1]
    exp = oracle_expect(g, xs, "float32", 4096, chunk_bytes=4096)
    _check_bytes(outs, exp, "allreduce", 2, 4096)
    # N = 2: a single commutative add -> also bit-exact to the definition (c5)
    _check_bytes(outs, definition.allreduce(xs, "float32"), "allreduce", 2, 4096)


ALGOS = [
    ("ring", "allreduce", 2, {}), ("ring", "allreduce", 3, {}), ("ring", "allreduce", 8, {}),
    ("ring", "allgather", 8, {}), ("ring", "reducescatter", 8, {}),
    ("dbt", "allreduce", 8, {}), ("hm", "allreduce", 8, {"g": 4}), ("hm", "allgather", 8, {"g": 4}),
    ("synth", "allgather", 8, {"seed": 0, "fanout": 2}), ("synth", "reducescatter", 8, {"seed": 3, "fanout": 3}),
]


def _inputs(coll, dtype, n, count, seed=1, mode="uniform"):
    m = count * n if coll == "reducescatter" else count
    return inp.all_inputs(dtype, seed, n, m, mode)


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
@pytest.mark.parametrize("dtype", ["float32", "bfloat16"])
def test_algorithms_bit_exact_vs_replay(name, coll, n, kw, dtype):
    """Several tiles, several micro-batches and instances, ragged tail."""
    g = oir.generate(name, coll, n, **kw)
    count = 3 * 4096 + 77
    text = _hdr(g, chunkbytes=4096, instances=2, fifodepth=2)
    xs = _inputs(coll, dtype, n, count)
    outs, info, err = run_virtual(R, text, coll, xs, dtype, count)
    assert err == 0
    exp = oracle_expect(g, xs, dtype, count, chunk_bytes=4096, instances=2, K=2)
    _check_bytes(outs, exp, coll, n, count)


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
def test_algorithms_int32_exact_vs_definition(name, coll, n, kw):
    g = oir.generate(name, coll, n, **kw)
    count = 10000
    text = _hdr(g, chunkbytes=8192, instances=3)
    xs = _inputs(coll, "int32", n, count, mode="wrap")
    outs, _, err = run_virtual(R, text, coll, xs, "int32", count)
    assert err == 0
    _check_bytes(outs, definition_expect(coll, xs, "int32"), coll, n, count)


@pytest.mark.parametrize("dtype", ["float16", "float32", "bfloat16", "int32"])
@pytest.mark.parametrize("op", ["sum", "max", "min"])
def test_dtypes_and_ops_ring(dtype, op):
    g = oir.ring_allreduce(4)
    count = 5000
    text = _hdr(g, chunkbytes=2048, instances=2)
    xs = _inputs("allreduce", dtype, 4, count)
    outs, _, err = run_virtual(R, text, "allreduce", xs, dtype, count, op=op)
    assert err == 0
    exp = oracle_expect(g, xs, dtype, count, op=op, chunk_bytes=2048, instances=2)
    _check_bytes(outs, exp, "allreduce", 4, count)


@pytest.mark.parametrize("name,coll,n,kw", ALGOS[2:8])
@pytest.mark.parametrize("dtype,rtol", [("float32", 1e-5), ("bfloat16", 2e-2)])
def test_tolerance_vs_naive_definition(name, coll, n, kw, dtype, rtol):
    """north_star: within 1e-5 (fp32) / 2e-2 (bf16) relative of naive-order summation,
    with the cancellation-safe bound |g - ref| <= rtol * sum_k |x_k|."""
    if coll == "allgather":
        pytest.skip("no arithmetic")
    g = oir.generate(name, coll, n, **kw)
    count = 20000
    xs = _inputs(coll, dtype, n, count, seed=5)
    outs, _, err = run_virtual(R, _hdr(g, chunkbytes=16384, instances=2), coll, xs, dtype, count)
    assert err == 0
    ref = definition_expect(coll, xs, dtype)
    den = definition.abs_sum(xs, dtype)
    for r in range(n):
        d = den if coll == "allreduce" else den[r * count:(r + 1) * count]
        diff = np.abs(numerics.to_f32(outs[r], dtype).astype(np.float64) -
                      numerics.to_f32(ref[r], dtype).astype(np.float64))
        assert np.all(diff <= rtol * d + 1e-30)


@pytest.mark.parametrize("coll", ["allreduce", "allgather", "reducescatter"])
@pytest.mark.parametrize("count", [1, 7, 8, 129, 4097])
def test_edge_counts_and_inplace(coll, count):
    """Tails: counts below N, not multiples of the vector width; in-place variants."""
    n = 8
    g = oir.generate("ring", coll, n)
    dtype = "bfloat16"
    xs = _inputs(coll, dtype, n, count, seed=9)
    for inplace in (False, True):
        outs, _, err = run_virtual(R, _hdr(g, chunkbytes=1024, instances=2), coll, xs, dtype, count,
                                   inplace=inplace)
        assert err == 0
        exp = oracle_expect(g, xs, dtype, count, chunk_bytes=1024, instances=2)
        _check_bytes(outs, exp, coll, n, count)


def test_count_zero_is_noop():
    import torch
    grp = R.VirtualGroup(4, 0)
    try:
        t = [torch.zeros(1, device="cuda:0") for _ in range(4)]
        for c in grp.comms:
            R.rescclAllReduce(t[0].data_ptr(), t[0].data_ptr(), 0, R.rescclFloat32, R.rescclSum, c.handle, 0)
        torch.cuda.synchronize()
    finally:
        grp.destroy()


def test_repeated_calls_monotone_flags():
    """Flags/counters are monotone across calls (no reset kernel): 5 back-to-back calls
    with different sizes reuse the FIFOs correctly."""
    import torch
    from gpu_helpers import to_numpy, to_torch
    n = 4
    g = oir.ring_allreduce(n)
    text = _hdr(g, chunkbytes=2048, instances=2, fifodepth=2)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(text)
        for it, count in enumerate([5000, 100, 9999, 4096, 1]):
            xs = _inputs("allreduce", "float32", n, count, seed=it)
            s = [to_torch(x, "float32") for x in xs]
            rv = [torch.empty_like(x) for x in s]
            grp.allreduce(s, rv)
            torch.cuda.synchronize()
            exp = oracle_expect(g, xs, "float32", count, chunk_bytes=2048, instances=2, K=2)
            _check_bytes([to_numpy(t, "float32") for t in rv], exp, "allreduce", n, count)
        assert grp.async_error() == 0
    finally:
        grp.destroy()


@pytest.mark.parametrize("budget", [1, 2, 4, 8, 16])
def test_tb_budget_sweep_hm_and_dbt(budget):
    """C3: DBT and HM 2x4 AllReduce under a TB budget; result independent of the plan."""
    for g in (oir.dbt_allreduce(8), oir.hm_allreduce(2, 4)):
        count = 40000
        text = _hdr(g, chunkbytes=8192, tbbudget=budget)
        xs = _inputs("allreduce", "bfloat16", 8, count, seed=budget)
        outs, info, err = run_virtual(R, text, "allreduce", xs, "bfloat16", count)
        assert err == 0
        assert max(info["blocks_per_rank"]) <= max(budget, max(info["ctas"]))
        exp = oracle_expect(g, xs, "bfloat16", count, chunk_bytes=8192, instances=info["instances"],
                            model=info["linkmodel"])
        _check_bytes(outs, exp, "allreduce", 8, count)


def test_load_rejects_bad_ir():
    grp = R.VirtualGroup(2, 0)
    try:
        with pytest.raises(R.ResCCLError):
            grp.comms[0].load("algo name=x coll=allreduce nranks=3 nchunks=3\n")
        with pytest.raises(R.ResCCLError):
            grp.comms[0].load("algo name=x coll=allreduce nranks=2 nchunks=2\nt 0 1 0 0 rrc\nt 1 0 0 0 rrc\n")
    finally:
        grp.destroy()


@pytest.mark.parametrize("name,coll,n,kw", ALGOS)
@pytest.mark.parametrize("dtype", ["bfloat16", "int32"])
def test_direct_transport_bit_exact(name, coll, n, kw, dtype):
    """Direct push/pull transport (R23) on virtual ranks: same bytes as the oracle."""
    g = oir.generate(name, coll, n, **kw)
    count = 3 * 4096 + 77
    text = _hdr(g, chunkbytes=4096, instances=2, direct=1)
    xs = _inputs(coll, dtype, n, count)
    outs, info, err = run_virtual(R, text, coll, xs, dtype, count)
    assert err == 0 and info["direct"] == 1
    exp = oracle_expect(g, xs, dtype, count, chunk_bytes=4096, instances=2, K=2)
    _check_bytes(outs, exp, coll, n, count)


@pytest.mark.parametrize("coll", ["allreduce", "allgather", "reducescatter"])
@pytest.mark.parametrize("count", [1, 129, 4097, 300001])
def test_direct_edge_counts_inplace(coll, count):
    n = 8
    g = oir.generate("ring", coll, n)
    xs = _inputs(coll, "bfloat16", n, count, seed=4)
    for inplace in (False, True):
        outs, _, err = run_virtual(R, _hdr(g, chunkbytes=65536, instances=3, direct=1), coll, xs, "bfloat16",
                                   count, inplace=inplace)
        assert err == 0
        exp = oracle_expect(g, xs, "bfloat16", count, chunk_bytes=65536, instances=3)
        _check_bytes(outs, exp, coll, n, count)


@pytest.mark.parametrize("name,coll,kw,fifo", [("synth", "reducescatter", {"seed": 0, "fanout": 2}, 2),
                                               ("synth", "reducescatter", {"seed": 0, "fanout": 2}, 1),
                                               ("synth", "reducescatter", {"seed": 1, "fanout": 2}, 2),
                                               ("ring", "allreduce", {}, 1),
                                               ("synth", "allgather", {"seed": 0, "fanout": 3}, 1)])
def test_direct_flag_rings_regression(name, coll, kw, fifo):
    """R26 regression: links fed by two sending lanes under the direct transport, several
    micro-batches, shallow flag rings (this hung before rings were split per lane)."""
    n = 8
    g = oir.generate(name, coll, n, **kw)
    count = 5 * 2048 + 13
    text = _hdr(g, chunkbytes=8192, instances=2, fifodepth=fifo, direct=1)
    xs = _inputs(coll, "float32", n, count, seed=5)
    outs, info, err = run_virtual(R, text, coll, xs, "float32", count)
    assert err == 0 and info["direct"] == 1
    exp = oracle_expect(g, xs, "float32", count, chunk_bytes=8192, instances=2, K=fifo)
    _check_bytes(outs, exp, coll, n, count)


@pytest.mark.parametrize("coll", ["allreduce", "allgather", "reducescatter"])
@pytest.mark.parametrize("direct", [0, 1])
def test_misaligned_bf16_pointers(coll, direct):
    """SURVEY d2 tails: bf16 buffers at 2-byte offsets (not 16-byte aligned) take the
    element path of the register mover and the unaligned TMA tails; bytes = the oracle's."""
    import torch
    from gpu_helpers import poison, to_numpy, to_torch
    n, dtype = 8, "bfloat16"
    g = oir.generate("ring", coll, n)
    text = _hdr(g, chunkbytes=1 << 20, instances=2, direct=direct, tmamin=4096)
    for count in (4097, 300001):
        xs = _inputs(coll, dtype, n, count, seed=6)
        grp = R.VirtualGroup(n, 0)
        try:
            grp.load(text)
            sends, recvs = [], []
            for r in range(n):
                base = torch.empty(xs[r].size + 1, dtype=torch.bfloat16, device="cuda:0")
                sends.append(base[1:])  # 2-byte offset
                sends[-1].copy_(to_torch(xs[r], dtype))
                m = count * n if coll == "allgather" else count
                out = torch.empty(m + 3, dtype=torch.bfloat16, device="cuda:0")
                poison(out)
                recvs.append(out[3:])  # 6-byte offset
            getattr(grp, coll)(sends, recvs)
            torch.cuda.synchronize()
            assert grp.async_error() == 0
            outs = [to_numpy(t, dtype) for t in recvs]
        finally:
            grp.destroy()
        exp = oracle_expect(g, xs, dtype, count, chunk_bytes=1 << 20, instances=2)
        _check_bytes(outs, exp, coll, n, count)


def test_count_2pow24_plus_3_direct_allreduce():
    """SURVEY d2 tail count 2^24 + 3 (bf16, 32 MiB per rank, TMA engine + ragged tail) on
    exactly representable inputs: every association order gives the definition's bits."""
    n, dtype, count = 8, "bfloat16", (1 << 24) + 3
    g = oir.generate("ring", "allreduce", n)
    text = _hdr(g, chunkbytes=8 << 20, instances=6, direct=1)
    xs = [inp.rank_input(dtype, 7, r, count, mode="exact") for r in range(n)]
    outs, _, err = run_virtual(R, text, "allreduce", xs, dtype, count)
    assert err == 0
    _check_bytes(outs, definition.allreduce(xs, dtype), "allreduce", n, count)


@pytest.mark.parametrize("coll", ["allreduce", "reducescatter"])
@pytest.mark.parametrize("dtype,op", [("bfloat16", "sum"), ("float32", "sum"), ("int32", "sum"),
                                      ("float16", "max"), ("float32", "max")])
@pytest.mark.parametrize("bulkred", [0, 1])
def test_inplace_tma_reduce_paths(coll, dtype, op, bulkred):
    """In-place reduce primitives on the TMA engine, with the combine warps (bulkred=0) or
    the L2 bulk reduction of the incoming tile (bulkred=1; f32 max keeps the combine path):
    bytes = the oracle's replay (one correctly rounded local (+) incoming per hop, R8)."""
    n = 8
    g = oir.generate("ring", coll, n)
    count = 40000 + 37
    text = _hdr(g, chunkbytes=1 << 20, instances=2, direct=1, tmamin=4096, bulkred=bulkred)
    xs = _inputs(coll, dtype, n, count, seed=8)
    outs, _, err = run_virtual(R, text, coll, xs, dtype, count, op=op, inplace=True)
    assert err == 0
    exp = oracle_expect(g, xs, dtype, count, op=op, chunk_bytes=1 << 20, instances=2)
    _check_bytes(outs, exp, coll, n, count)


@pytest.mark.parametrize("name,coll,kw", [("ring", "allreduce", {}), ("hm", "allreduce", {"g": 2}),
                                          ("ring", "allgather", {}), ("dbt", "allreduce", {})])
@pytest.mark.parametrize("tmamin", [4096, 1 << 30])
def test_cuda_graph_capture_and_replay(name, coll, kw, tmamin):
    """Device-side flag epochs (devepoch=1): collectives captured into a CUDA graph replay
    correctly, interleaved with eager calls of the same plan (the epochs the graph's
    kernels read advance on the device)."""
    import torch
    from gpu_helpers import to_numpy, to_torch
    n, count, dtype = 4, 30000 + 5, "int32"
    g = oir.generate(name, coll, n, **kw)
    text = _hdr(g, chunkbytes=1 << 16, instances=2, direct=1, tmamin=tmamin)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(text)
        ref_in = [_inputs(coll, dtype, n, count, seed=s) for s in (21, 22)]
        s = [to_torch(x, dtype) for x in ref_in[0]]
        m = count * n if coll == "allgather" else count
        r = [torch.zeros(m, dtype=torch.int32, device="cuda:0") for _ in range(n)]
        f = getattr(grp, coll)
        f(s, r)  # eager warm-up (compiles the kernel outside the capture)
        torch.cuda.synchronize()
        st = torch.cuda.Stream()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=st):
            f(s, r, stream=st)
            f(s, r, stream=st)
        for it in range(3):
            x = ref_in[it % 2]
            for t, v in zip(s, x):
                t.copy_(to_torch(v, dtype))
            for t in r:
                t.zero_()
            graph.replay()
            torch.cuda.synchronize()
            assert grp.async_error() == 0
            outs = [to_numpy(t, dtype) for t in r]
            _check_bytes(outs, definition_expect(coll, x, dtype), coll, n, count)
            f(s, r)  # an eager call between replays advances the same epochs
            torch.cuda.synchronize()
            _check_bytes([to_numpy(t, dtype) for t in r], definition_expect(coll, x, dtype), coll, n, count)
    finally:
        grp.destroy()


def test_graph_capture_refused_with_host_epochs():
    """devepoch=0 keeps host-side epochs: capture is refused with InvalidUsage before any
    CUDA state changes, and the communicator stays usable."""
    import torch
    from gpu_helpers import to_torch
    n, count = 2, 4096
    text = _hdr(oir.generate("ring", "allreduce", n), devepoch=0)
    grp = R.VirtualGroup(n, 0)
    try:
        grp.load(text)
        xs = _inputs("allreduce", "float32", n, count)
        s = [to_torch(x, "float32") for x in xs]
        r = [torch.empty_like(t) for t in s]
        st = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with pytest.raises(R.ResCCLError) as e:
            with torch.cuda.graph(g, stream=st):
                grp.allreduce(s, r)
        assert e.value.code == R.rescclInvalidUsage
    finally:
        grp.destroy()
    outs, _, err = run_virtual(R, text, "allreduce", xs, "float32", count)
    assert err == 0
    _check_bytes(outs, definition.allreduce(xs, "float32"), "allreduce", n, count)


@pytest.mark.parametrize("dtype", ["bfloat16", "float16"])
@pytest.mark.parametrize("tma", [0, 1])
def test_16bit_add_all_bit_patterns(dtype, tma):
    """Packed 16-bit adds (add.rn.bf16x2 / add.rn.f16x2) against the correctly rounded sum
    on (almost) every finite bit pattern -- subnormals, ties, signed zeros included: two
    ranks, one add per element, so the definition's single rounding is the exact answer."""
    import numpy as np
    n = 2
    pats = np.arange(1 << 16, dtype=np.uint32).astype(np.uint16)
    if dtype == "bfloat16":
        f = numerics.bf16_to_f32(pats)
    else:
        f = pats.view(np.float16).astype(np.float32)
    keep = np.isfinite(f) & (np.abs(f) < (2.0 ** 100 if dtype == "bfloat16" else 16384.0))
    a = pats[keep]
    rng = np.random.default_rng(11)
    b = a[rng.permutation(a.size)]
    xs = [a.copy(), b.copy()]
    if dtype == "float16":
        xs = [x.view(np.float16) for x in xs]
    count = xs[0].size
    g = oir.generate("ring", "allreduce", n)
    text = _hdr(g, chunkbytes=1 << 20, instances=2, direct=1, tmamin=4096 if tma else 1 << 30)
    outs, _, err = run_virtual(R, text, "allreduce", xs, dtype, count)
    assert err == 0
    _check_bytes(outs, definition.allreduce(xs, dtype), "allreduce", n, count)
