"""REDUCE_SUM_ACCURATE: fp32 with per-thread fp32 Neumaier
pairs then fp64 above the thread, and fp64 with double-double accumulation,
checked against the EXACT sum (math.fsum via oracle/ref.py):
|r - S| <= u|S| + E*sum|x| with u the output unit roundoff and E the
accumulation error: (L+1)^2 * 2^-48 for fp32 (compensated fp32 chains of
length <= L, then fp64), (L+1) * 2^-100 for double-double; L is the variant's
chain length (tests/_chain.py, computed from the launch shape).  Plus cancellation pins a plain
sum fails, special values, every grid combine, segmented and host entry."""
import math

import numpy as np
import pytest

from oracle import ref
import oracle
import synth
from tests._util import to_device
from tests._chain import checked_chain

pytestmark = pytest.mark.gpu


def _rb():
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    return rb


def _gate(dtype, S, A, L):
    if dtype == "float32":
        return 2.0 ** -24 * abs(S) + (L + 1) ** 2 * 2.0 ** -48 * A + 1e-300
    return 2.0 ** -53 * abs(S) + (L + 1) * 2.0 ** -100 * A + 1e-300


def _check(x, r, plan):
    S = ref.sum_fp(x)
    if not math.isfinite(S):
        assert (math.isnan(S) and math.isnan(r)) or r == S, (S, r)
        return
    A = ref.abs_sum(x)
    err = abs(float(r) - S)
    L = checked_chain(x.dtype.name, "sum_accurate", plan)  # test-side chain, not the library's
    assert err <= _gate(x.dtype.name, S, A, L), (x.dtype.name, x.size, r, S, err, L, plan)


VARIANTS = [dict(), dict(mode="deterministic"), dict(grid_combine=0, block=256), dict(grid_combine=2),
            dict(grid_combine=3), dict(grid_combine=4, grid=16), dict(stage="smem", unroll=8, block=256),
            dict(block_combine=3, block=128), dict(grid=148, grid_combine=3), dict(grid_combine=5),
            dict(grid_combine=5, block=32, unroll=1)]


@pytest.mark.parametrize("dtype", ["float32", "float64"])
@pytest.mark.parametrize("dist", ["uniform01", "uniform_pm1"])
def test_accurate_sum_vs_exact(dtype, dist):
    rb = _rb()
    for k, n in enumerate([1, 7, 1000, 4097, (1 << 18) + 5, (1 << 21) + 3]):
        x = synth.make(dtype, n, dist, 900 + k)
        t = to_device(x, k % 4)
        for v in VARIANTS:
            r = rb.reduce(t, "sum_accurate", **v).item()
            _check(x, r, rb.query_plan(dtype, "sum_accurate", n, in_ptr=t.data_ptr(), **v))


def test_accurate_fp32_atomic_variants():
    rb = _rb()
    x = synth.make("float32", (1 << 20) + 9, "uniform_pm1", 4)
    t = to_device(x, 1)
    for v in (dict(grid_combine=1), dict(block_combine=1), dict(block_combine=2, block=128)):
        r = rb.reduce(t, "sum_accurate", **v).item()
        _check(x, r, rb.query_plan("float32", "sum_accurate", x.size, in_ptr=t.data_ptr(), **v))


def test_accurate_fp64_rejects_atomic_combines():
    rb = _rb()
    import torch
    t = torch.ones(1000, dtype=torch.float64, device="cuda")
    for v in (dict(grid_combine=1), dict(block_combine=1)):
        with pytest.raises(rb.ReduceError):
            rb.reduce(t, "sum_accurate", **v)
    with pytest.raises(rb.ReduceError):
        rb.reduce(torch.ones(10, dtype=torch.int32, device="cuda"), "sum_accurate")


def test_cancellation_pins():
    """Plain element-type accumulation loses these; the accurate sum must not."""
    rb = _rb()
    import torch
    # fp64: 1e16 + 1 - 1e16 + 1 = 2 exactly (a plain fp64 sum gives 0 or 1)
    base = np.array([1e16, 1.0, -1e16, 1.0], np.float64)
    x = np.tile(base, 1 << 16)  # 2^18 elements, exact sum 2^17
    for v in VARIANTS:
        assert rb.reduce(to_device(x), "sum_accurate", **v).item() == float(1 << 17), v
    # fp32: 2^24 + 1 + 1 + ... (2^20 ones) - 2^24  -> exactly 2^20 (fp32 plain sums drop the ones)
    y = np.ones((1 << 20) + 2, np.float32)
    y[0], y[-1] = 2.0 ** 24, -(2.0 ** 24)
    for v in VARIANTS:
        assert rb.reduce(to_device(y), "sum_accurate", **v).item() == float(1 << 20), v


@pytest.mark.parametrize("dtype", ["float32", "float64"])
def test_accurate_special_values(dtype):
    rb = _rb()
    sp = lambda k: synth.special_f(dtype, k)
    for kinds in (["nan"], ["inf"], ["ninf"], ["inf", "ninf"], ["neg_nan"]):
        x = synth.make(dtype, 100003, "uniform_pm1", 1)
        for i, k in enumerate(kinds):
            x[13 + 50000 * i] = sp(k)
        for v in VARIANTS[:6]:
            r = rb.reduce(to_device(x, 1), "sum_accurate", **v).item()
            S = ref.sum_fp(x)
            assert (math.isnan(S) and math.isnan(r)) or r == S, (kinds, v, r, S)


def test_accurate_segmented_and_host():
    rb = _rb()
    import torch
    x = synth.make("float64", 200000, "uniform_pm1", 8)
    offs = np.array([0, 0, 1, 33, 4097, 100000, 200000], np.int64)
    got = rb.reduce_segmented(torch.from_numpy(x).cuda(), torch.from_numpy(offs).cuda(), "sum_accurate").cpu().numpy()
    for i in range(len(offs) - 1):
        seg = x[offs[i]:offs[i + 1]]
        S, A = ref.sum_fp(seg), ref.abs_sum(seg)
        assert abs(got[i] - S) <= _gate("float64", S, A, 64), (i, got[i], S)
    xf = synth.make("float32", (1 << 24) + 7, "uniform01", 3)
    r = rb.reduce_host(xf, "sum_accurate")
    S = oracle.reduce(xf, "sum")
    assert abs(float(r) - S.value) <= _gate("float32", S.value, S.abs_sum, 64)
