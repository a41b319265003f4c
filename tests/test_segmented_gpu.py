"""Segmented / batched reduction against the oracle applied to
every segment: bit-exact for int32 and min/max, G1 + G2 for fp sums (chain of a
warp- or block-per-segment reduction).  Empty, single-element, misaligned and
skewed (power-law) segments; warp and block groups; uniform batches."""
import math

import numpy as np
import pytest

import oracle
import synth
from tests._util import NP, BITS

pytestmark = pytest.mark.gpu
DTYPES = ["int32", "float32", "float64"]
OPS = ["sum", "min", "max"]


def _chain(length, dtype, lanes):
    # per-thread: m vectors through a lane tree (depth log2 VE) into 2 accumulators
    # (or one accumulator per lane), + head/tail, + merge; then group / block combines
    ve = 4 if dtype == "float64" else 8
    m = math.ceil(length / (ve * lanes))
    return m + int(math.log2(ve)) + 3 + 5 + (5 if lanes > 32 else 0)


def _check_segments(x, bounds, op, got, lanes):
    dt = x.dtype.name
    for i, (lo, hi) in enumerate(bounds):
        seg = x[lo:hi]
        ref = oracle.reduce(seg, op)
        if dt == "int32" or op != "sum":
            g = int(got[i:i + 1].view(BITS[dt])[0])
            assert g == ref.bits, (dt, op, i, lo, hi, got[i], ref.value)
        else:
            ok, msg = oracle.check_sum(float(got[i]), ref, seg.dtype, max(hi - lo, 1),
                                       chain=_chain(hi - lo, dt, lanes))
            assert ok, (dt, i, lo, hi, msg)


def _segments(rng, nseg, max_len, skew=False):
    if skew:  # power-law lengths: a few huge segments, many tiny ones
        lens = np.minimum((rng.pareto(1.2, nseg) * 16).astype(np.int64), max_len)
    else:
        lens = rng.integers(0, max_len + 1, nseg)
    lens[::7] = 0
    lens[1::11] = 1
    offs = np.zeros(nseg + 1, np.int64)
    offs[1:] = np.cumsum(lens)
    return offs


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("group", [0, 1, 2, 3])
@pytest.mark.parametrize("skew", [False, True])
def test_segmented_matches_oracle_per_segment(dtype, group, skew):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(17 + group))
    offs = _segments(rng, 3000, 5000, skew)
    total = int(offs[-1])
    x = synth.make(dtype, total + 3, "int_full" if dtype == "int32" else "uniform_pm1", 5)[3:]
    xt = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    ot = torch.from_numpy(offs).cuda()
    bounds = list(zip(offs[:-1].tolist(), offs[1:].tolist()))
    lanes = {0: 32, 1: 32, 2: 256, 3: 8}[group]
    for op in OPS:
        got = rb.reduce_segmented(xt, ot, op, seg_group=group).cpu().numpy()
        _check_segments(x, bounds, op, got, lanes)


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("rows,cols", [(1, 1), (7, 33), (1000, 1024), (64, 100003), (4096, 17), (100003, 64),
                                       (3000, 129)])
def test_batched_rows(dtype, rows, cols):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    x = synth.make(dtype, rows * cols, "int_full" if dtype == "int32" else "uniform01", rows + cols)
    xt = torch.from_numpy(x).cuda().view(rows, cols)
    bounds = [(r * cols, (r + 1) * cols) for r in range(rows)]
    for group in (0, 1, 2, 3):
        auto = 8 if cols <= 128 else (32 if cols <= 4096 else 256)
        lanes = {0: auto, 1: 32, 2: 256, 3: 8}[group]
        for op in OPS:
            got = rb.reduce_batched(xt, op, seg_group=group).cpu().numpy()
            _check_segments(x, bounds, op, got, lanes)


def test_segmented_special_values_and_determinism():
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    x = synth.make("float32", 100000, "uniform_pm1", 9)
    x[5] = np.nan
    x[50000] = np.inf
    x[70000] = -0.0
    offs = np.array([0, 10, 10, 50001, 70000, 70001, 100000], np.int64)
    xt, ot = torch.from_numpy(x).cuda(), torch.from_numpy(offs).cuda()
    bounds = list(zip(offs[:-1].tolist(), offs[1:].tolist()))
    for group in (1, 2, 3):
        for op in OPS:
            got = rb.reduce_segmented(xt, ot, op, seg_group=group).cpu().numpy()
            _check_segments(x, bounds, op, got, {1: 32, 2: 256, 3: 8}[group])
    outs = {rb.reduce_segmented(xt, ot, "sum").cpu().numpy().tobytes() for _ in range(20)}
    assert len(outs) == 1
