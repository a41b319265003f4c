"""Histogram on the GPU against oracle.histogram, bit-exact:
int32 bins are exact integer arithmetic on both sides; fp32 bins are decided
in fp32 on both sides by the rule DESIGN.md R13 defines,
floor(fl32(fl32(x - lo_f) * scale)) -- a definition chosen for the kernel (the
paper only motivates histograms), itself pinned against the
exact-rational bins on non-power-of-two grids by tests/test_oracle.py.  Shared-memory and global-memory bin paths, ragged
head/tail, out-of-range values, NaN/inf, large inputs."""
import numpy as np
import pytest

import oracle
import synth
from tests._util import to_device

pytestmark = pytest.mark.gpu


def _rb():
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    return rb


@pytest.mark.parametrize("dtype", ["int32", "float32"])
@pytest.mark.parametrize("nbins", [1, 7, 256, 1000, 16384, 16385, 100000, 1 << 20])
def test_histogram_bit_exact(dtype, nbins):
    rb = _rb()
    for k, n in enumerate([0, 1, 13, 4097, (1 << 20) + 3]):
        if dtype == "int32":
            x = synth.make("int32", n, "int_small", 40 + k)
            lo, hi = -900.0, 1000.0 - 7 * k
        else:
            x = synth.make("float32", n, "uniform_pm1", 40 + k)
            lo, hi = -0.75, 0.8 + 0.01 * k
        t = to_device(x, k % 8)
        got = rb.histogram(t, lo, hi, nbins).cpu().numpy().view(np.uint32)
        want = oracle.histogram(x, lo, hi, nbins)
        assert (got == want).all(), (dtype, nbins, n, np.nonzero(got != want)[0][:5])


def test_histogram_special_values_and_big():
    rb = _rb()
    x = synth.make("float32", (1 << 24) + 5, "uniform01", 3)
    x[[0, 5, 99, -1]] = [np.nan, np.inf, -np.inf, -0.0]
    t = to_device(x, 3)
    for nbins in (10, 4096, 65536):
        got = rb.histogram(t, 0.0, 1.0, nbins).cpu().numpy().view(np.uint32)
        want = oracle.histogram(x, 0.0, 1.0, nbins)
        assert (got == want).all()
        assert int(got.sum()) == int(((x >= 0) & (x < 1)).sum())


@pytest.mark.parametrize("lo,hi,nbins", [
    (-2.0 ** 31, 2.0 ** 31, 1000),        # range * nbins >= 2^32: 64-bit quotient path
    (-2.0 ** 32, 2.0 ** 32, 1 << 20),     # widest accepted range, many bins (bin-range passes)
    (-65536.0, 65537.0, 65535),           # range * nbins just above 2^32
    (-65536.0, 0.0, 65535),               # range * nbins just below 2^32: 32-bit path
    (0.0, 3.0, 3),                        # one bin per value
    (5.0, 6.0, 1),                        # range 1 (the zero multiplier)
    (5.0, 6.0, 3),                        # range 1, more bins than values
    (-512.0, 512.0, 64),                  # power-of-two range (multiplier 1)
    (-513.0, 512.0, 64),                  # 2^k + 1
    (-511.0, 512.0, 1000),                # 2^k - 1, range * nbins near 2^20
    (-40000.0, 67000.0, 40000),           # range * nbins just below 2^32, odd divisor
    (2.0 ** 31 - 10, 2.0 ** 31 + 10, 4),  # narrow, hi above INT32_MAX: clamped 32-bit range check
    (-2.0 ** 31 - 10, -2.0 ** 31 + 10, 3),  # narrow, lo below INT32_MIN
    (2.0 ** 31 + 5, 2.0 ** 31 + 100, 7),  # entirely above the int32 range: nothing counted
    (-2.0 ** 32, -2.0 ** 31 - 1, 2),      # entirely below
])
def test_histogram_int32_wide_ranges(lo, hi, nbins):
    rb = _rb()
    x = synth.make("int32", (1 << 20) + 11, "int_full", 77)
    x[:6] = [np.iinfo(np.int32).min, np.iinfo(np.int32).max, 0, -1, 1, 2]
    edge = np.arange(-12, 12, dtype=np.int64)  # values next to both ends of the int32 range
    x[1000:1024] = (edge + 2 ** 31).astype(np.int64).clip(-2 ** 31, 2 ** 31 - 1).astype(np.int32)
    x[2000:2024] = (edge - 2 ** 31).clip(-2 ** 31, 2 ** 31 - 1).astype(np.int32)
    if hi - lo < 2 ** 20:
        y = (x[7::3].astype(np.int64) % int(2 * (hi - lo))) + int(lo) - int((hi - lo) // 2)
        x[7::3] = y.clip(-2 ** 31, 2 ** 31 - 1).astype(np.int32)
    t = to_device(x, 5)
    got = rb.histogram(t, lo, hi, nbins).cpu().numpy().view(np.uint32)
    want = oracle.histogram(x, lo, hi, nbins)
    assert (got == want).all(), np.nonzero(got != want)[0][:5]


@pytest.mark.parametrize("dtype", ["int32", "float32"])
def test_histogram_replication_boundaries(dtype):
    """bins per block at the shared-copy boundaries (32, 16, ... copies per bin)"""
    rb = _rb()
    n = (1 << 19) + 5
    x = synth.make(dtype, n, "int_small" if dtype == "int32" else "uniform01", 91)
    lo, hi = (-1000.0, 1001.0) if dtype == "int32" else (0.0, 1.0)
    for nbins in (2, 31, 32, 33, 511, 512, 513, 1023, 1024, 2048, 4095, 4096, 8192, 16383):
        t = to_device(x, nbins % 8)
        got = rb.histogram(t, lo, hi, nbins).cpu().numpy().view(np.uint32)
        want = oracle.histogram(x, lo, hi, nbins)
        assert (got == want).all(), (nbins, np.nonzero(got != want)[0][:5])


@pytest.mark.parametrize("dtype", ["int32", "float32"])
@pytest.mark.parametrize("nbins", [16385, 65536, 100003])
def test_histogram_16bit_counters_carry(dtype, nbins):
    """16384 < nbins: one pass with 16-bit shared counters.  A few bins get far
    more than 2^15 elements per block (every 0x8000 moves to the global count),
    neighbours of those bins (same shared word) stay exact, and the rest is
    spread over every bin."""
    rb = _rb()
    n = (1 << 25) + 13
    if dtype == "int32":
        x = synth.make("int32", n, "int_full", 5) % nbins
        x[: n // 2] = 7            # bin 7 (word 3, high half) and
        x[n // 2: n // 2 + n // 4] = 6  # bin 6, the low half of the same word
        lo, hi = 0.0, float(nbins)
    else:
        x = synth.make("float32", n, "uniform01", 5)
        x[: n // 2] = np.float32(0.5)
        x[n // 2: n // 2 + n // 4] = np.float32(0.5) - np.float32(1.0 / nbins)
        lo, hi = 0.0, 1.0
    t = to_device(x, 1)
    got = rb.histogram(t, lo, hi, nbins).cpu().numpy().view(np.uint32)
    want = oracle.histogram(x, lo, hi, nbins)
    assert (got == want).all(), np.nonzero(got != want)[0][:5]
    assert int(got.sum()) == int(want.sum())


@pytest.mark.parametrize("nbins", [16385, 65535, 65536])
def test_histogram_16bit_merge_aligned_and_misaligned_counts(nbins):
    """The 16-bit path merges a shared word's two halves with one 64-bit global
    add when `counts` is 8-byte aligned (and n < 2^32), else with two 32-bit
    adds; an odd nbins leaves the last word's high half without a bin (the
    64-bit add must not touch counts[nbins]).  Both layouts, a sentinel past
    the end, and counts that are not zero on entry (the call overwrites them)."""
    import torch
    rb = _rb()
    n = (1 << 22) + 5
    x = synth.make("float32", n, "uniform01", 61)
    x[:1000] = np.float32(1.0 - 1e-7)  # the last bin gets a heavy count
    t = to_device(x, 3)
    want = oracle.histogram(x, 0.0, 1.0, nbins)
    for off in (0, 1):  # counts 8-byte aligned, then 4 bytes past alignment
        buf = torch.full((nbins + 4,), 12345, dtype=torch.int32, device="cuda")
        counts = buf[off:off + nbins]
        rb.histogram(t, 0.0, 1.0, nbins, counts=counts)
        got = counts.cpu().numpy().view(np.uint32)
        assert (got == want).all(), (nbins, off, np.nonzero(got != want)[0][:5])
        assert int(buf[off + nbins].item()) == 12345  # nothing written past the end


def test_histogram_back_to_back_and_graphs():
    """Every call overwrites `counts` whatever they held: back-to-back calls on
    one stream with different bin counts and grid sizes (the replicated 32-bit,
    bin-range and 16-bit paths), garbage in `counts` on entry, inputs rewritten
    by torch kernels right before each call, reduce() calls interleaved, and a
    captured graph replayed with fresh inputs."""
    import torch
    rb = _rb()
    s = torch.cuda.Stream()
    cases = [(256, 0), (1000, 1), (65536, 4097), (40000, 1 << 20), (7, 13), (16384, (1 << 21) + 3), (256, 1 << 22)]
    with torch.cuda.stream(s):
        rb.prepare(s, 1 << 22)
        xs = [torch.empty(n, dtype=torch.float32, device="cuda") for _, n in cases]
        outs = [torch.full((nb,), -7, dtype=torch.int32, device="cuda") for nb, _ in cases]
        for it in range(3):
            hosts = []
            for k, ((nb, n), xt) in enumerate(zip(cases, xs)):
                x = synth.make("float32", n, "uniform_pm1", 700 + 10 * it + k)
                xt.copy_(torch.from_numpy(x).to("cuda", non_blocking=False))
                xt.mul_(1.0)  # a torch kernel writes the input right before the histogram
                outs[k].fill_(12345)
                rb.histogram(xt, -0.9, 0.95, nb, counts=outs[k], stream=s)
                rb.reduce(xt, "max", stream=s) if n else None
                hosts.append(x)
            s.synchronize()
            for (nb, n), x, o in zip(cases, hosts, outs):
                want = oracle.histogram(x, -0.9, 0.95, nb)
                got = o.cpu().numpy().view(np.uint32)
                assert (got == want).all(), (it, nb, n, np.nonzero(got != want)[0][:5])
        # graph: two histograms captured, replayed with new inputs
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            rb.histogram(xs[2], -0.9, 0.95, 65536, counts=outs[2], stream=s)
            rb.histogram(xs[6], -0.9, 0.95, 256, counts=outs[6], stream=s)
        for rep in range(3):
            x2 = synth.make("float32", xs[2].numel(), "uniform_pm1", 900 + rep)
            x6 = synth.make("float32", xs[6].numel(), "uniform_pm1", 950 + rep)
            xs[2].copy_(torch.from_numpy(x2))
            xs[6].copy_(torch.from_numpy(x6))
            outs[2].fill_(-1)
            outs[6].fill_(-1)
            g.replay()
            s.synchronize()
            assert (outs[2].cpu().numpy().view(np.uint32) == oracle.histogram(x2, -0.9, 0.95, 65536)).all(), rep
            assert (outs[6].cpu().numpy().view(np.uint32) == oracle.histogram(x6, -0.9, 0.95, 256)).all(), rep



@pytest.mark.parametrize("nbins", [1, 3, 256, 1000, 16384, 16385, 65536, 100000, 131072])
def test_histogram_f32_bin_edges(nbins):
    """The shared-memory kernels compute an fp32 bin as the bits of
    fl_rz(t + 2^23) minus those of 2^23 (t = fl(fl(x - lo) * scale)) instead of a
    float-to-int conversion; x < lo must wrap out of range and x >= hi / NaN be
    forced out.  Elements at and one ulp around lo, hi and every sampled bin
    edge, -0.0 with lo = 0, subnormals, +-inf, NaN, on two ranges (bit-exact
    against the oracle's rule, DESIGN R13)."""
    rb = _rb()
    rng = np.random.Generator(np.random.PCG64(77 + nbins))
    for lo, hi in ((0.0, 1.0), (-3.25, 11.5)):
        lo32, hi32 = np.float32(lo), np.float32(hi)
        k = np.unique(np.concatenate([np.arange(min(nbins, 64)), rng.integers(0, nbins + 1, 2000)]))
        edges = (lo32 + (k.astype(np.float64) * (hi - lo) / nbins)).astype(np.float32)
        vals = [edges, np.nextafter(edges, np.float32(-np.inf)), np.nextafter(edges, np.float32(np.inf)),
                np.array([lo32, hi32, np.nextafter(lo32, np.float32(-1e30)), np.nextafter(hi32, np.float32(-1e30)),
                          np.nextafter(hi32, np.float32(1e30)), np.float32(-0.0), np.float32(1e-45),
                          np.float32(-1e-45), np.float32(np.inf), np.float32(-np.inf), np.float32(np.nan)],
                         dtype=np.float32)]
        x = np.concatenate(vals).astype(np.float32)
        x = np.concatenate([x, rng.uniform(lo - 1, hi + 1, 300_000).astype(np.float32)])
        rng.shuffle(x)
        t = to_device(x, 5)
        got = rb.histogram(t, lo, hi, nbins).cpu().numpy().view(np.uint32)
        want = oracle.histogram(x, lo, hi, nbins)
        assert (got == want).all(), (nbins, lo, hi, np.nonzero(got != want)[0][:5])
