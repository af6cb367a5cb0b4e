"""f3 (NVLS transport), CPU side: the oracle's NVLS schedule pinned to the collective
definitions and to invariants I1/I3/I6, the AR partition's closed form, and the C ABI's
host-only NVLS entry points (NVRTC build of every kernel variant, argument errors)."""
import numpy as np
import pytest

import resccl_inputs as inp
from oracle import definition, nvls

COLLS = ["allreduce", "reducescatter", "allgather"]


@pytest.mark.parametrize("coll", COLLS)
@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 8])
def test_symbolic_invariants(coll, n):
    st = nvls.symbolic(coll, n)  # raises on I1 (overlap) / I6 (undefined read)
    for r in range(n):
        for c in range(n):
            got = st.get((r, c))
            if coll == "allreduce":
                assert got == set(range(n))  # I3: every rank holds the full sum
            elif coll == "allgather":
                assert got == {c}  # I3: <r,c> = rank c's block
            elif c == r:
                assert got == set(range(n))  # RS: rank r owns the reduced chunk r


def test_symbolic_catches_a_dropped_primitive():
    """A schedule missing one mred leaves a rank without the full result (I3 fails)."""
    st = nvls.symbolic("allreduce", 4)
    assert all(st[(r, c)] == {0, 1, 2, 3} for r in range(4) for c in range(4))
    orig = nvls.schedule
    try:
        nvls.schedule = lambda coll, n: [p for p in orig(coll, n) if p != ("mred", 2, 2)]
        st2 = nvls.symbolic("allreduce", 4)
        assert st2[(0, 2)] == {2}
    finally:
        nvls.schedule = orig


@pytest.mark.parametrize("nbytes", [0, 4, 16, 28, 64, 1000, 4096 * 3 + 8, (1 << 20) + 4])
@pytest.mark.parametrize("n", [1, 2, 3, 8])
def test_ar_partition_closed_form(nbytes, n):
    parts = nvls.ar_partition(nbytes, n)
    assert parts[0][0] == 0 and parts[-1][1] == nbytes
    for (lo, hi), (lo2, _) in zip(parts, parts[1:]):
        assert hi == lo2  # contiguous, disjoint cover
    sl = -(-nbytes // n)
    for lo, hi in parts:
        assert (lo % 16 == 0 or lo == hi == nbytes) and 0 <= hi - lo <= sl + 15


@pytest.mark.parametrize("coll", COLLS)
@pytest.mark.parametrize("n", [1, 2, 3, 8])
@pytest.mark.parametrize("count", [2, 6, 1000, 4098])
def test_replay_equals_definition_int32(coll, n, count):
    xs = [inp.rank_input("int32", 3, r, count * (n if coll == "reducescatter" else 1)) for r in range(n)]
    xs[0][0] = 0x7FFFFFFF  # wraparound
    out = nvls.replay(coll, xs, "int32")
    ref = {"allreduce": lambda: definition.allreduce(xs, "int32"),
           "reducescatter": lambda: definition.reducescatter(xs, "int32"),
           "allgather": lambda: definition.allgather(xs)}[coll]()
    for a, b in zip(out, ref):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("dtype", ["float32", "float16", "bfloat16"])
@pytest.mark.parametrize("op", ["sum", "max", "min"])
def test_replay_equals_definition_exact_fp(dtype, op):
    n, count = 8, 4096 + 2
    xs = [inp.rank_input(dtype, 1, r, count, mode="exact") for r in range(n)]
    out = nvls.replay("allreduce", xs, dtype, op)
    ref = definition.allreduce(xs, dtype, op)
    for a, b in zip(out, ref):
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))


def test_eligibility_rule():
    assert nvls.eligible("allreduce", 2, "bfloat16", "sum")
    assert not nvls.eligible("allreduce", 3, "bfloat16", "sum")  # half a 4-byte granule
    assert nvls.eligible("allreduce", 3, "float32", "sum")
    assert not nvls.eligible("allreduce", 4, "float32", "max")  # no f32 max in multimem
    assert nvls.eligible("allreduce", 4, "int32", "min")
    assert nvls.eligible("allgather", 7, "int32", "sum")
    assert not nvls.eligible("allreduce", 4, "int32", "sum", send_off=2)
    assert not nvls.eligible("allgather", 4, "float16", "sum", recv_off=6)


@pytest.mark.parametrize("coll", COLLS)
@pytest.mark.parametrize("dtype", ["int32", "float32", "float16", "bfloat16"])
def test_nvls_kernels_build_for_sm100a(coll, dtype):
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    for op in ("sum", "max", "min"):
        assert R.rescclCompileNvls(coll, dtype, op) > 0


def test_nvls_abi_argument_errors():
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    with pytest.raises(R.ResCCLError) as e:
        R.rescclNvlsSupported(0)
    assert e.value.code == R.rescclInvalidArgument
    with pytest.raises(R.ResCCLError) as e:
        R.rescclNvlsAllocAll([], 1 << 20)
    assert e.value.code == R.rescclInvalidArgument
    with pytest.raises(R.ResCCLError) as e:
        R.rescclNvlsFree(0, 0)
    assert e.value.code == R.rescclInvalidArgument
    with pytest.raises(R.ResCCLError) as e:
        R.rescclNvlsAlloc(0, 1 << 20, lambda b: [b])
    assert e.value.code == R.rescclInvalidArgument


def test_nvls_option_in_plan_info():
    import paper_conf_sigcomm_liuhlgcwz025_b200 as R
    text = R.rescclGenerateIr("ring", "allreduce", 4)
    info = R.rescclPlanIr(text, "nvls=1 nvlsctas=8")
    assert info["nvls"] == 1 and info["nvlsctas"] == 8
    assert R.rescclPlanIr(text)["nvls"] == 0
    with pytest.raises(R.ResCCLError):
        R.rescclPlanIr(text, "nvlsctas=0")
