"""Segmented / batched reduction against the oracle applied to
every segment: bit-exact for int32 and min/max, G1 + G2 for fp sums (chain of a
warp- or block-per-segment reduction).  Empty, single-element, misaligned and
skewed (power-law) segments; warp and block groups; uniform batches."""
import math

import numpy as np
import pytest

import oracle
import synth
from tests._util import NP, BITS, to_device

pytestmark = pytest.mark.gpu
DTYPES = ["int32", "float32", "float64"]
OPS = ["sum", "min", "max"]


def _chain(length, dtype, lanes):
    # per-thread: m vectors through a lane tree (depth log2 VE) into 2 accumulators
    # (or one accumulator per lane), + head/tail, + merge; then group / block combines
    ve = 4 if dtype == "float64" else 8
    if lanes < 0:  # element-balanced chunks: <= 4*VE elements in order per lane, lane scan,
        el = 4 * ve  # then the chunk pieces joined 32 at a time by warp butterflies
        return min(length, el) + 1 + 5 + 1 + math.ceil(math.ceil(length / (32 * el) + 1) / 32) * 6 + 2
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
@pytest.mark.parametrize("group", [0, 1, 2, 3, 4])
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
    lanes = {0: -1, 1: 32, 2: 256, 3: 8, 4: 1}[group]
    for op in OPS:
        got = rb.reduce_segmented(xt, ot, op, seg_group=group).cpu().numpy()
        _check_segments(x, bounds, op, got, lanes)


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("rows,cols", [(1, 1), (7, 33), (1000, 1024), (64, 100003), (4096, 17), (100003, 64),
                                       (3000, 129), (50001, 8), (30001, 32), (1001, 56), (2, 64)])
def test_batched_rows(dtype, rows, cols):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    x = synth.make(dtype, rows * cols, "int_full" if dtype == "int32" else "uniform01", rows + cols)
    xt = torch.from_numpy(x).cuda().view(rows, cols)
    bounds = [(r * cols, (r + 1) * cols) for r in range(rows)]
    s = x.dtype.itemsize
    for group in (0, 1, 2, 3, 4):
        rb_ = cols * s
        auto = 1 if rb_ <= 512 else (8 if rb_ <= 4096 else (32 if rb_ <= 16384 else 256))
        lanes = {0: auto, 1: 32, 2: 256, 3: 8, 4: 1}[group]
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
    for group in (1, 2, 3, 5):
        for op in OPS:
            got = rb.reduce_segmented(xt, ot, op, seg_group=group).cpu().numpy()
            _check_segments(x, bounds, op, got, {1: 32, 2: 256, 3: 8, 5: -1}[group])
    outs = {rb.reduce_segmented(xt, ot, "sum").cpu().numpy().tobytes() for _ in range(20)}
    assert len(outs) == 1


def _skewed(rng, nseg, huge):
    """many short segments (0..40 elements) with a few huge ones (up to `huge`
    elements) at seeded positions: the long-segment queue's workload"""
    lens = rng.integers(0, 41, nseg)
    pos = rng.choice(nseg, 6, replace=False)
    lens[pos] = [huge, huge // 3, 70000, 16385, 4099, 300]
    offs = np.zeros(nseg + 1, np.int64)
    offs[1:] = np.cumsum(lens)
    return offs


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("group", [0, 1, 2, 3, 4])
def test_segmented_long_segments_load_balanced(dtype, group):
    """segments far longer than a group's first round go through the chunk
    queue (k_seg_chunks / k_seg_finish); results per segment vs the oracle,
    and bitwise identical over repeated calls (fixed chunk order)"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(101 + group))
    offs = _skewed(rng, 20000, 3_000_001)
    total = int(offs[-1])
    x = synth.make(dtype, total + 5, "int_full" if dtype == "int32" else "uniform_pm1", 12)[5:]
    xt = to_device(x, 3)
    ot = torch.from_numpy(offs).cuda()
    bounds = list(zip(offs[:-1].tolist(), offs[1:].tolist()))
    lanes = {0: -1, 1: 32, 2: 256, 3: 8, 4: 1}[group]
    for op in OPS + (["sum_accurate"] if dtype != "int32" else []):
        got = rb.reduce_segmented(xt, ot, op, seg_group=group)
        if op == "sum_accurate":
            g = got.cpu().numpy()
            for i in np.nonzero(np.diff(offs) > 1000)[0]:
                lo, hi = bounds[i]
                exact = math.fsum(x[lo:hi].astype(np.float64))
                a = float(np.abs(x[lo:hi].astype(np.float64)).sum())
                assert abs(float(g[i]) - exact) <= 2.0 ** -23 * abs(exact) + 1e-9 * a, (i, g[i], exact)
            continue
        _check_segments(x, bounds, op, got.cpu().numpy(), lanes)
        again = rb.reduce_segmented(xt, ot, op, seg_group=group)
        assert got.cpu().numpy().tobytes() == again.cpu().numpy().tobytes()


def test_segmented_queue_overflow_falls_back():
    """more queued chunks than the queue holds (kSegQItems = 2^18): the
    segments that do not fit are finished by their own group, results exact"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    nseg = 150000
    lens = np.full(nseg, 8 * 40, np.int64)  # 40 vectors: queued by 1-lane groups (2 items each)
    lens[::1000] = 70000                     # a few multi-chunk ones
    offs = np.zeros(nseg + 1, np.int64)
    offs[1:] = np.cumsum(lens)
    x = synth.make("int32", int(offs[-1]), "int_full", 13)
    xt, ot = torch.from_numpy(x).cuda(), torch.from_numpy(offs).cuda()
    got = rb.reduce_segmented(xt, ot, "sum", seg_group=4).cpu().numpy()
    want = np.add.reduceat(x.astype(np.int64), offs[:-1]).astype(np.int64)
    want = ((want + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
    assert (got == want).all(), np.nonzero(got != want)[0][:5]
    gmax = rb.reduce_segmented(xt, ot, "max", seg_group=4).cpu().numpy()
    assert (gmax == np.maximum.reduceat(x, offs[:-1])).all()


def test_batched_long_rows_chunked():
    """a few rows of millions of elements: every row is cut into chunks"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rows, cols = 3, 5_000_003
    x = synth.make("float64", rows * cols, "intvalued", 14)
    xt = torch.from_numpy(x).cuda().view(rows, cols)
    for group in (0, 1, 2, 3, 4):
        got = rb.reduce_batched(xt, "sum", seg_group=group).cpu().numpy()
        want = x.reshape(rows, cols).astype(np.float64).sum(axis=1)  # integer-valued: exact in any order
        assert (got == want).all(), (group, got, want)


def test_segmented_graph_capture_with_queue():
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(5))
    offs = _skewed(rng, 5000, 1_000_000)
    x = synth.make("float32", int(offs[-1]), "uniform01", 15)
    xt, ot = torch.from_numpy(x).cuda(), torch.from_numpy(offs).cuda()
    ref = rb.reduce_segmented(xt, ot, "sum").cpu().numpy()
    s = torch.cuda.Stream()
    rb.prepare(s, 1 << 20)
    out = torch.empty(len(offs) - 1, dtype=torch.float32, device="cuda")
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        rb.reduce_segmented(xt, ot, "sum", out=out, stream=s)
    for _ in range(4):
        out.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert out.cpu().numpy().tobytes() == ref.tobytes()


@pytest.mark.parametrize("group", [0, 1, 2, 3, 4])
def test_segmented_decreasing_pairs_are_empty(group):
    """include/reduce.h: a decreasing offsets pair is an empty segment (the
    identity), including next to long (queued) segments and overlapping ranges"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    x = synth.make("int32", 300_000, "int_full", 21)
    offs = np.array([0, 100, 50, 200_000, 150_000, 150_001, 299_999, 10, 300_000], np.int64)
    xt, ot = torch.from_numpy(x).cuda(), torch.from_numpy(offs).cuda()
    ident = {"sum": 0, "min": np.iinfo(np.int32).max, "max": np.iinfo(np.int32).min}
    for op in OPS:
        got = rb.reduce_segmented(xt, ot, op, seg_group=group).cpu().numpy()
        for i in range(len(offs) - 1):
            lo, hi = int(offs[i]), int(offs[i + 1])
            want = oracle.reduce(x[lo:hi], op).value if hi > lo else ident[op]
            assert int(got[i]) == int(want), (op, i, lo, hi, got[i], want)


@pytest.mark.parametrize("dtype", DTYPES)
def test_batched_aligned_short_rows_vs_misaligned(dtype):
    """rows of whole 32-byte vectors on 32-byte boundaries (<= 256 B) take the
    one-thread-per-row kernel with all loads in flight; the same rows starting
    one element off 32-byte alignment take the group kernel -- both exact"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    ve = 4 if dtype == "float64" else 8
    for nv in (1, 3, 8):
        cols, rows = nv * ve, 20011
        x = synth.make(dtype, rows * cols + 1, "int_full" if dtype == "int32" else "intvalued", nv)
        for off in (0, 1):
            xt = to_device(x[off:off + rows * cols], off).view(rows, cols)
            for op in OPS:
                got = rb.reduce_batched(xt, op).cpu().numpy()
                _check_segments(x[off:off + rows * cols], [(r * cols, (r + 1) * cols) for r in range(rows)], op, got, 1)


AUTO_TILED_MIN_KB = 1 / 32  # reduce_api.cpp kTiledAutoMinLv: auto takes every eligible row size


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("row_kb,rows", [(1, 1), (1, 33), (2, 4099), (4, 17), (4, 1000), (8, 9), (16, 5), (32, 3),
                                         (32, 40), (64, 2048), (96, 2051), (1 / 32, 1), (1 / 32, 1027),
                                         (1 / 16, 515), (1 / 8, 4097), (1 / 4, 3001), (1 / 2, 129)])
def test_batched_tiled_rows(dtype, row_kb, rows):
    """seg_group 6 (k_rows_tiled): 32 KB tiles of whole 1-32 KB rows, including
    a partial last tile; bit-exact (int32, min/max) or G1 + G2 (fp sums) per row,
    the auto choice identical, the fixed tree reproducible, special values."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    s = np.dtype(NP[dtype]).itemsize
    cols = int(row_kb * 1024) // s
    x = synth.make(dtype, rows * cols, "int_full" if dtype == "int32" else "uniform_pm1", int(31 * row_kb) + rows)
    if dtype != "int32" and rows > 3:
        # indexed per row (rows may be as short as 4 elements: fp64 32 B rows)
        x[cols + min(5, cols - 1)] = np.nan          # row 1: NaN
        x[2 * cols + min(7, cols - 1)] = -np.inf     # row 2: -inf
        x[3 * cols:4 * cols] = 0.0
        x[3 * cols + min(2, cols - 1)] = -0.0        # row 3: all zeros with one -0.0
    xt = torch.from_numpy(x).cuda().view(rows, cols)
    bounds = [(r * cols, (r + 1) * cols) for r in range(rows)]
    ops = OPS + (["sum_accurate"] if dtype != "int32" else [])
    for op in ops:
        got = rb.reduce_batched(xt, op, seg_group=6).cpu().numpy()
        if op == "sum_accurate":  # the exact sum and test_accurate_gpu's gate (chain <= 64)
            from oracle import ref as exact
            from tests.test_accurate_gpu import _gate
            for i, (lo, hi) in enumerate(bounds):
                S = exact.sum_fp(x[lo:hi])
                r = float(got[i])
                if not math.isfinite(S):
                    assert (math.isnan(S) and math.isnan(r)) or r == S, (i, r, S)
                else:
                    assert abs(r - S) <= _gate(dtype, S, exact.abs_sum(x[lo:hi]), 64), (op, i, r, S)
        else:
            _check_segments(x, bounds, op, got, 32)
        again = rb.reduce_batched(xt, op, seg_group=6).cpu().numpy()
        assert got.tobytes() == again.tobytes(), op
        acc_f32_mid = op == "sum_accurate" and dtype == "float32" and 1 / 8 <= row_kb <= 1 / 2  # auto keeps the old kernel
        if row_kb >= AUTO_TILED_MIN_KB and not acc_f32_mid:  # auto takes the same kernel
            assert rb.reduce_batched(xt, op).cpu().numpy().tobytes() == got.tobytes(), op


def test_batched_tiled_rows_rejects_ineligible():
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    x = torch.zeros(64 * 1024 + 8, dtype=torch.float32, device="cuda")
    with pytest.raises(rb.ReduceError):  # 3 KB rows
        rb.reduce_batched(x[:48 * 768].view(48, 768), "sum", seg_group=6)
    with pytest.raises(rb.ReduceError):  # rows of whole 32 KB tiles, but too few of them
        rb.reduce_batched(x[:4 * 16384].view(4, 16384), "sum", seg_group=6)
    with pytest.raises(rb.ReduceError):  # misaligned start
        rb.reduce_batched(x[1:1 + 64 * 256].view(64, 256), "sum", seg_group=6)
    # ineligible rows under auto still take the group kernels
    got = rb.reduce_batched(x[1:1 + 64 * 256].view(64, 256), "sum").cpu().numpy()
    assert (got == 0).all()
