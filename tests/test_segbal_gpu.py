"""Element-balanced segmented reduction (reduce_segmented on an offsets array,
csrc/reduce_segbal.cuh) against the oracle applied to every
segment: bit-exact for int32 and min/max, G1 + G2 for fp sums.

The cases aim at the chunk machinery: segments shorter than a lane, longer
than a chunk (4 KB) and spanning hundreds of chunks, boundaries exactly on
lane / chunk edges, runs of empty segments (including more than a chunk's
offsets list holds: the walk path), offsets[0] > 0 and offsets[-1] < len(x),
every input misalignment, non-monotone offsets (the per-segment fallback) and
bitwise determinism over repeated calls and CUDA-graph replays."""
import math

import numpy as np
import pytest

import oracle
from oracle import ref
import synth
from tests._util import BITS, to_device
from tests.test_segmented_gpu import _chain

pytestmark = pytest.mark.gpu
DTYPES = ["int32", "float32", "float64"]
KINDS = ["ones", "tiny", "lane", "chunk", "chunk_pm1", "long"]


def _ops(dtype):
    return ["sum", "min", "max"] + (["sum_accurate"] if dtype != "int32" else [])


def _data(dtype, n, seed):
    return synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", seed)


def _check(x, offs, op, got):
    dt = x.dtype.name
    ident = oracle.reduce(x[:0], "min" if op == "min" else ("max" if op == "max" else "sum"))
    for i in range(len(offs) - 1):
        lo, hi = int(offs[i]), int(offs[i + 1])
        if hi <= lo:
            if dt == "int32" or op in ("min", "max"):
                assert int(got[i:i + 1].view(BITS[dt])[0]) == ident.bits, (op, i, "empty")
            else:
                assert float(got[i]) == 0.0, (op, i, "empty")
            continue
        seg = x[lo:hi]
        if op == "sum_accurate":  # test_accurate_gpu's gate, L = the balanced chain
            S, A = ref.sum_fp(seg), ref.abs_sum(seg)
            L = _chain(hi - lo, dt, -1)
            tol = (2.0 ** -24 * abs(S) + (L + 1) ** 2 * 2.0 ** -48 * A if dt == "float32"
                   else 2.0 ** -53 * abs(S) + (L + 1) * 2.0 ** -100 * A)
            if not math.isfinite(S):
                assert (math.isnan(S) and math.isnan(got[i])) or got[i] == S, (i, S, got[i])
            else:
                assert abs(float(got[i]) - S) <= tol, (i, lo, hi, got[i], S)
            continue
        want = oracle.reduce(seg, op)
        if dt == "int32" or op != "sum":
            g = int(got[i:i + 1].view(BITS[dt])[0])
            assert g == want.bits, (dt, op, i, lo, hi, got[i], want.value)
        else:
            ok, msg = oracle.check_sum(float(got[i]), want, seg.dtype, hi - lo, chain=_chain(hi - lo, dt, -1))
            assert ok, (dt, i, lo, hi, msg)


def _run(x_np, offs, dtype, misalign=0, groups=(0, 5), ops=None):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    xt = to_device(x_np, misalign)
    ot = torch.from_numpy(np.asarray(offs, np.int64)).cuda()
    for group in groups:
        for op in ops or _ops(dtype):
            got = rb.reduce_segmented(xt, ot, op, seg_group=group)
            g = got.cpu().numpy()
            _check(x_np, offs, op, g)
            again = rb.reduce_segmented(xt, ot, op, seg_group=group).cpu().numpy()
            assert g.tobytes() == again.tobytes(), (op, "not deterministic")


def _offsets(lens, start=0):
    offs = np.zeros(len(lens) + 1, np.int64)
    offs[0] = start
    offs[1:] = start + np.cumsum(lens)
    return offs


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("misalign", [0, 1, 3, 7])
def test_powerlaw_lengths(dtype, misalign):
    rng = np.random.Generator(np.random.PCG64(2019 + misalign))
    lens = np.minimum((rng.pareto(1.2, 20000) * 12.8).astype(np.int64) + 1, 400_000)
    lens[::13] = 0
    offs = _offsets(lens)
    x = _data(dtype, int(offs[-1]), 31 + misalign)
    _run(x, offs, dtype, misalign)


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", KINDS)
def test_length_regimes(dtype, kind):
    """lengths around the lane (8 vectors) and chunk (8 KB) sizes, so
    boundaries fall on lane and chunk edges and pieces cross both"""
    rng = np.random.Generator(np.random.PCG64(KINDS.index(kind)))
    el = 16 if dtype == "float64" else 32  # elements per lane (4 x 32 bytes); chunk = 32 lanes = 4 KB
    c = 32 * el
    if kind == "ones":
        lens = np.ones(30000, np.int64)
    elif kind == "tiny":
        lens = rng.integers(0, 4, 30000)
    elif kind == "lane":
        lens = rng.choice([el - 1, el, el + 1, 2 * el], 3000)
    elif kind == "chunk":
        lens = np.full(300, c, np.int64)
    elif kind == "chunk_pm1":
        lens = rng.choice([c - 1, c, c + 1, 3 * c + 5], 300)
    else:
        lens = np.array([5, 1_000_003, 17, 250 * c, 0, 3, c * 33 + 1], np.int64)
    offs = _offsets(lens)
    x = _data(dtype, int(offs[-1]) + 9, 7)
    _run(x, offs, dtype, misalign=int(rng.integers(0, 8)))


@pytest.mark.parametrize("dtype", DTYPES)
def test_offsets_window_and_empty_runs(dtype):
    """offsets[0] > 0, offsets[-1] < len(x); a run of 5000 empty segments in
    one chunk (more entries than its shared list holds: the walk path) and
    shorter runs elsewhere; empty first and last segments"""
    rng = np.random.Generator(np.random.PCG64(77))
    lens = rng.integers(0, 200, 8000)
    lens[3000:8000:2] = 0
    lens[100:5100] = 0
    lens[6000:6010] = 0
    lens[0] = 0
    lens[-1] = 0
    offs = _offsets(lens, start=12345)
    x = _data(dtype, int(offs[-1]) + 777, 8)
    _run(x, offs, dtype, misalign=5)
    lens2 = np.concatenate([rng.integers(1, 50, 100), np.zeros(6000, np.int64), rng.integers(1, 50, 100)])
    offs2 = _offsets(lens2, start=3)
    x2 = _data(dtype, int(offs2[-1]) + 3, 9)
    _run(x2, offs2, dtype, misalign=2, ops=["sum", "max"])


def test_all_empty_and_single():
    x = _data("float32", 5000, 3)
    _run(x, np.array([10, 10, 10, 10], np.int64), "float32")
    _run(x, np.array([4999, 5000], np.int64), "float32")
    _run(x, np.array([0, 5000], np.int64), "float32")
    _run(x, np.array([0, 1, 2, 3, 4999, 5000], np.int64), "float32", misalign=1)


@pytest.mark.parametrize("dtype", DTYPES)
def test_special_values(dtype):
    if dtype == "int32":
        pytest.skip("no special values")
    x = _data(dtype, 300_000, 4)
    x[5] = np.nan
    x[70_000] = np.inf
    x[70_001] = -np.inf
    x[120_000] = -0.0
    x[150_000:150_010] = 0.0
    x[150_004] = -0.0
    x[200_000] = np.inf
    offs = np.array([0, 4, 6, 50_000, 70_001, 70_002, 120_000, 120_001, 150_000, 150_010, 200_001, 300_000],
                    np.int64)
    _run(x, offs, dtype, ops=["sum", "min", "max"])


def test_non_monotone_offsets_fall_back():
    """a decreasing pair is an empty segment and later segments may overlap
    earlier ones: the chunk kernel reduces one segment per warp instead"""
    x = _data("int32", 300_000, 21)
    offs = np.array([0, 100, 50, 200_000, 150_000, 150_001, 299_999, 10, 300_000], np.int64)
    _run(x, offs, "int32", groups=(0, 5))
    # and the next monotone call on the same stream is balanced again (flag reset)
    lens = np.random.Generator(np.random.PCG64(3)).integers(0, 3000, 400)
    offs2 = _offsets(lens)
    _run(_data("int32", int(offs2[-1]), 22), offs2, "int32")


def test_graph_capture_and_replay():
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(5))
    lens = np.minimum((rng.pareto(1.2, 50000) * 12.8).astype(np.int64) + 1, 1 << 20)
    offs = _offsets(lens)
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


def test_matches_group_kernels_exactly_for_ints():
    """int32 results are order-independent: the balanced path and every group
    kernel give the same bits on the same skewed input"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(11))
    lens = np.minimum((rng.pareto(1.1, 40000) * 10).astype(np.int64), 2_000_000)
    offs = _offsets(lens, start=1)
    x = _data("int32", int(offs[-1]) + 1, 12)
    xt, ot = to_device(x, 1), torch.from_numpy(offs).cuda()
    for op in ("sum", "min", "max"):
        outs = {rb.reduce_segmented(xt, ot, op, seg_group=g).cpu().numpy().tobytes() for g in (0, 1, 2, 3, 4, 5)}
        assert len(outs) == 1, op


def _reduceat(x, offs, op):
    """numpy reference per segment (vectorised; empty segments -> identity)."""
    x = x[: int(offs[-1])]  # reduceat's last segment runs to the end of its input
    lo = offs[:-1]
    empty = offs[1:] <= lo
    idx = np.minimum(lo, max(x.size - 1, 0))
    if op == "sum":
        r = np.add.reduceat(x.astype(np.int64 if x.dtype == np.int32 else np.float64), idx)
        r[empty] = 0
        return r
    f = np.minimum if op == "min" else np.maximum
    r = f.reduceat(x, idx)
    ident = {"min": np.iinfo(np.int32).max, "max": np.iinfo(np.int32).min} if x.dtype == np.int32 else \
        {"min": np.inf, "max": -np.inf}
    r[empty] = ident[op]
    return r


@pytest.mark.parametrize("dtype", ["int32", "float32"])
def test_bench_workload_full_size(dtype):
    """bench.py's `segmented` workload at full size (1 M power-law segments over
    ~60 M elements, the launch the bench times): int32 sums (mod 2^32), int32 /
    fp32 min and max bit-exact against numpy reduceat; fp32 sums within the
    G2 gate per segment ((L + 1) u sum|x|, L the balanced chain)."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(2019 + 1000 * 6))
    total = (256 << 20) // 4
    nseg = total // 64
    lens = np.minimum((rng.pareto(1.2, nseg) * 64 * 0.2).astype(np.int64) + 1, 1 << 20)
    offs = np.minimum(np.concatenate([[0], np.cumsum(lens)]), total)
    n = int(offs[-1])
    x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform01", 66)
    xt, ot = torch.from_numpy(x).cuda(), torch.from_numpy(offs).cuda()
    for op in ("sum", "min", "max"):
        got = rb.reduce_segmented(xt, ot, op).cpu().numpy()
        want = _reduceat(x, offs, op)
        if dtype == "int32" and op == "sum":
            want = ((want + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
            assert (got == want).all(), np.nonzero(got != want)[0][:5]
        elif op == "sum":
            lens_ = np.diff(offs)
            absum = np.abs(want)  # uniform01: all terms >= 0, sum|x| = sum
            el = 32
            chain = np.minimum(lens_, el) + 8 + 6 * (np.ceil(np.ceil(lens_ / (32 * el) + 1) / 32)) + 2
            gate = (chain + 1) * 2.0 ** -24 * absum + 2.0 ** -24 * absum  # + the final fp32 rounding
            err = np.abs(got.astype(np.float64) - want)
            assert (err <= gate).all(), (np.nonzero(err > gate)[0][:5], err.max())
        else:
            assert (got.view(np.uint32) == want.astype(x.dtype).view(np.uint32)).all(), op


def test_concurrent_streams_independent_workspaces():
    """two streams run balanced segmented calls at the same time: each stream's
    chunk arrays (and flags / tickets) are its own"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(44))
    cases = []
    for k in range(2):
        lens = np.minimum((rng.pareto(1.2, 30000) * 12.8).astype(np.int64) + 1, 300_000)
        offs = _offsets(lens, start=k)
        x = _data("int32", int(offs[-1]) + 1, 50 + k)
        cases.append((x, offs, to_device(x, k), torch.from_numpy(offs).cuda()))
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    for s in streams:
        rb.prepare(s, 1 << 20)
    outs = [torch.empty(len(c[1]) - 1, dtype=torch.int32, device="cuda") for c in cases]
    torch.cuda.synchronize()
    for rep in range(5):
        for (x, offs, xt, ot), s, o in zip(cases, streams, outs):
            rb.reduce_segmented(xt, ot, "sum", out=o, stream=s)
    torch.cuda.synchronize()
    for (x, offs, xt, ot), o in zip(cases, outs):
        want = _reduceat(x, offs, "sum")
        want = ((want + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
        assert (o.cpu().numpy() == want).all()


@pytest.mark.parametrize("lead", [0, 1, 5, 37])
def test_many_segments_scan_instances(lead):
    """Segment counts that select the scan kernel's K = 1 / 4 / 8 segments per
    thread (nseg up to ~1.6 M), with `lead` empty segments first, runs of 3-11
    empty segments that straddle the scan threads' K-segment groups, a segment
    spanning many warp ranges and single-element segments: every range start
    the scan claims (once per thread, round 2) must be the non-empty segment
    holding the range's first element.  int32 sum (mod 2^32) / max bit-exact
    against numpy reduceat, misaligned input."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    rng = np.random.Generator(np.random.PCG64(500 + lead))
    for nseg in (200_000, 700_000, 1_600_000):
        lens = rng.integers(1, 40, nseg)
        lens[:lead] = 0
        for start in rng.integers(lead, nseg - 20, 300):  # empty runs of 3..11
            lens[start:start + rng.integers(3, 12)] = 0
        lens[nseg // 2] = 3_000_000  # one segment across many ranges
        lens[nseg // 3: nseg // 3 + 5000] = 1
        offs = np.concatenate([[7], 7 + np.cumsum(lens)])
        n = int(offs[-1]) + 5
        x = synth.make("int32", n, "int_full", 70 + lead)
        xt = torch.empty(n + 1, dtype=torch.int32, device="cuda")[1:]
        xt.copy_(torch.from_numpy(x))
        ot = torch.from_numpy(offs).cuda()
        for op in ("sum", "max"):
            got = rb.reduce_segmented(xt, ot, op).cpu().numpy()
            want = _reduceat(x, offs, op)
            if op == "sum":
                want = ((want + 2 ** 31) % 2 ** 32 - 2 ** 31).astype(np.int32)
            assert (got == want.astype(np.int32)).all(), (nseg, op, np.nonzero(got != want)[0][:5])
