"""Host-buffer collectives through the C ABI (include/resccl.h, "Host buffers"): the
library stages host send / receive buffers through device memory, AllReduce in pieces
of RESCCL_HOST_PIECE bytes.  Results are compared byte for byte with the oracle: a
staged call is the device collective on the same bytes, and a piecewise AllReduce is
one AllReduce per piece (each piece its own chunk layout, reading R6), so the
expectation is the concatenation of the oracle's replays of the pieces."""
import os

import numpy as np
import pytest

import resccl_inputs as inp
from oracle import definition, ir as oir

from gpu_helpers import oracle_expect, run_virtual

pytestmark = pytest.mark.gpu

R = None


@pytest.fixture(scope="module", autouse=True)
def _lib():
    global R
    import paper_conf_sigcomm_liuhlgcwz025_b200 as mod
    R = mod


def _text(coll, n, **kw):
    g = oir.generate("ring", coll, n)
    for k, v in kw.items():
        g.extra[k] = str(v)
    return g, g.to_text()


def _inputs(coll, dtype, n, count, seed):
    return inp.all_inputs(dtype, seed, n, count * n if coll == "reducescatter" else count)


def _same(outs, exp):
    for r, (a, b) in enumerate(zip(outs, exp)):
        assert a.shape == b.shape, (r, a.shape, b.shape)
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8)), f"rank {r} differs"


@pytest.mark.parametrize("coll", ["allreduce", "allgather", "reducescatter"])
@pytest.mark.parametrize("where", [("pinned", "pinned"), ("pinned", "cuda:0"), ("cuda:0", "pinned"),
                                   ("cpu", "cpu")])
@pytest.mark.parametrize("inplace", [False, True])
def test_host_buffers_bit_exact(coll, where, inplace):
    send_dev, recv_dev = where
    if inplace and send_dev != recv_dev:
        pytest.skip("in-place buffers live in one place")
    n, count, dtype = 8, 4097, "bfloat16"
    g, text = _text(coll, n, chunkbytes=4096, instances=2)
    xs = _inputs(coll, dtype, n, count, seed=21)
    outs, _, err = run_virtual(R, text, coll, xs, dtype, count, inplace=inplace, send_dev=send_dev,
                               recv_dev=recv_dev)
    assert err == 0
    _same(outs, oracle_expect(g, xs, dtype, count, chunk_bytes=4096, instances=2))


def _piece_expect(g, coll, xs, dtype, count, pe, n, **kw):
    """Concatenation of the oracle's replays of the pieces [lo, lo+m) of the per-rank
    count: AR / AG inputs are column slices of each rank's buffer, RS inputs the column
    slice of each of its N rows; AG outputs interleave back into N rows."""
    cols = []
    for lo in range(0, count, pe):
        m = min(pe, count - lo)
        if coll == "reducescatter":
            ins = [np.concatenate([x[q * count + lo:q * count + lo + m] for q in range(n)]) for x in xs]
        else:
            ins = [x[lo:lo + m] for x in xs]
        cols.append((m, oracle_expect(g, ins, dtype, m, **kw)))
    if coll != "allgather":
        return [np.concatenate([c[r] for _, c in cols]) for r in range(n)]
    return [np.concatenate([np.concatenate([c[r][q * m:(q + 1) * m] for m, c in cols]) for q in range(n)])
            for r in range(n)]


@pytest.mark.parametrize("coll,dtype", [("allreduce", "float32"), ("allreduce", "bfloat16"), ("allreduce", "int32"),
                                        ("allgather", "bfloat16"), ("reducescatter", "float32"),
                                        ("reducescatter", "bfloat16")])
@pytest.mark.parametrize("where", [("pinned", "pinned"), ("pinned", "cuda:0"), ("cuda:0", "pinned")])
def test_host_collectives_in_pieces(coll, dtype, where, monkeypatch):
    """RESCCL_HOST_PIECE = 8 KiB: the call runs as 4 pieces (the last ragged), each
    bit-exact to the oracle's replay of that piece (AG outputs and RS inputs move as N
    strided rows).  A device-side AG output / RS input runs as one piece.  int32 AR also
    equals the definition."""
    send_dev, recv_dev = where
    n = 8
    elt = 2 if dtype == "bfloat16" else 4
    pe = 8192 // elt
    count = 3 * pe + 513
    monkeypatch.setenv("RESCCL_HOST_PIECE", str(8192))
    g, text = _text(coll, n, chunkbytes=2048, instances=2)
    xs = _inputs(coll, dtype, n, count, seed=5)
    one_piece = (coll == "allgather" and recv_dev == "cuda:0") or (coll == "reducescatter" and send_dev == "cuda:0")
    kw = dict(chunk_bytes=2048, instances=2)
    exp = oracle_expect(g, xs, dtype, count, **kw) if one_piece else _piece_expect(g, coll, xs, dtype, count, pe, n, **kw)
    for inplace in ((False, True) if send_dev == recv_dev else (False,)):
        outs, _, err = run_virtual(R, text, coll, xs, dtype, count, inplace=inplace, send_dev=send_dev,
                                   recv_dev=recv_dev)
        assert err == 0
        _same(outs, exp)
        if dtype == "int32":
            _same(outs, definition.allreduce(xs, dtype))


def test_host_buffers_refuse_graph_capture():
    import torch
    grp = R.VirtualGroup(2, 0)
    try:
        grp.load(_text("allreduce", 2)[1])
        h = torch.ones(1024).pin_memory()
        st = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with pytest.raises(R.ResCCLError):
            with torch.cuda.graph(g, stream=st):
                R.rescclAllReduce(h.data_ptr(), h.data_ptr(), 1024, R.rescclFloat32, R.rescclSum,
                                  grp.comms[0].handle, st.cuda_stream)
    finally:
        torch.cuda.synchronize()
        grp.destroy()
