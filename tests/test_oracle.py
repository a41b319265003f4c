"""Pins for the CPU oracle (no GPU).  Each test checks oracle/ against something
other than itself: closed forms, the paper's worked example, exact big-integer /
math.fsum arithmetic (oracle/ref.py), brute-force permutations, special values.
Pin ids P1..P11 follow SURVEY.md section 8(c) / DESIGN.md "Pins"."""
import math
import os
import random
import struct

import numpy as np
import pytest

import oracle
from oracle import ref, paper_codelets as pc
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
I32_MAX, I32_MIN = 2 ** 31 - 1, -(2 ** 31)


def f32bits(v):
    return struct.unpack("<I", struct.pack("<f", v))[0]


def f64bits(v):
    return struct.unpack("<Q", struct.pack("<d", v))[0]


# ------------------------------------------------------------ P1 closed forms
@pytest.mark.parametrize("n", [0, 1, 7, 1000, 1 << 20, (1 << 20) + 3])
@pytest.mark.parametrize("dtype", ["int32", "float32", "float64"])
def test_p1_ones(n, dtype):
    x = synth.make(dtype, n, "ones", 0)
    r = oracle.reduce(x, "sum")
    assert r.value == n
    if dtype != "int32":
        assert r.abs_sum == n


# ------------------------------------------------------------ P2 iota
@pytest.mark.parametrize("n", [0, 1, 2, 5793, 65536, 100000, (1 << 20) + 1])
def test_p2_iota_int32_wraps(n):
    x = synth.make("int32", n, "iota", 0)
    exact = (n * (n - 1) // 2) % (1 << 32)
    exact = exact - (1 << 32) if exact >= (1 << 31) else exact
    assert int(oracle.reduce(x, "sum").value) == exact


@pytest.mark.parametrize("n", [5793, 1 << 16, (1 << 22) + 5])
@pytest.mark.parametrize("dtype", ["float32", "float64"])
def test_p2_iota_fp(n, dtype):
    # oracle carries S in double: exact for n <= 2^27 (values < 2^24 are exact in fp32)
    x = synth.make(dtype, n, "iota", 0)
    assert oracle.reduce(x, "sum").value == n * (n - 1) // 2


# ------------------------------------------------------------ P3 integer-valued
@pytest.mark.parametrize("dtype,bound,n", [("float32", 1 << 7, 1 << 17), ("float64", 1 << 20, 1 << 18)])
def test_p3_integer_valued_fp_exact(dtype, bound, n):
    x = synth.make(dtype, n, "intvalued", 11, bound=bound)
    exact = sum(int(v) for v in x.astype(np.int64))
    r = oracle.reduce(x, "sum")
    assert r.value == exact
    assert r.abs_sum == sum(abs(int(v)) for v in x.astype(np.int64))


# ------------------------------------------------------------ int32 wrap
def test_int32_wraparound_pins():
    assert oracle.reduce(np.array([I32_MAX, 1], np.int32), "sum").value == I32_MIN
    assert oracle.reduce(np.array([I32_MIN, -1], np.int32), "sum").value == I32_MAX
    assert oracle.reduce(np.array([I32_MIN, I32_MIN], np.int32), "sum").value == 0


# ------------------------------------------------------------ P5 permutations
@pytest.mark.parametrize("dtype", ["int32", "float32", "float64"])
@pytest.mark.parametrize("n", [1, 2, 33, 4097, 1 << 16])
def test_p5_permutation_minmax(dtype, n):
    x = synth.make(dtype, n, "perm", 5 + n)
    assert oracle.reduce(x, "min").value == 0
    assert oracle.reduce(x, "max").value == n - 1
    # extremes at the ends
    x[[0, -1]] = x[[-1, 0]]
    assert oracle.reduce(x, "min").value == 0
    assert oracle.reduce(x, "max").value == n - 1


# ------------------------------------------------------------ P6 paper example
def _read_golden(name):
    rows = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, _, rest = line.partition(":") if ":" in line else line.partition(" ")
            rows[key.strip()] = [int(v) for v in rest.split()]
    return rows


def test_p6_fig1c_worked_example():
    g = _read_golden("fig1c_tree.txt")
    xs = g["input"]
    ms = g["max_size"][0]
    trace = []
    total = pc.codelet_cooperative(xs, max_size=ms, trace=trace)
    for vid, steps in trace:
        for s, row in enumerate(steps, start=1):
            assert row == g[f"vector {vid} step {s}"], (vid, s, row)
    assert [steps[-1][0] for _, steps in trace] == g["partials"]
    assert total == g["total"][0]
    # Fig. 3(a)/(b) reach the same total
    assert pc.codelet_va1(xs) == g["total"][0]
    assert pc.codelet_va2(xs, max_size=ms) == g["total"][0]
    # and so does the plain-definition oracle
    assert oracle.reduce(np.array(xs, np.int32), "sum").value == g["total"][0]


def test_p7_fig2_partial_warp():
    g = _read_golden("fig2_partial_warp.txt")
    n = g["n"][0]
    xs = list(range(1, n + 1))
    assert g["threads_per_vector"] == [32, n - 32]
    arr = np.array(xs, np.int32)
    assert oracle.reduce(arr, "sum").value == g["sum"][0]
    assert oracle.reduce(arr, "min").value == g["min"][0]
    assert oracle.reduce(arr, "max").value == g["max"][0]
    assert pc.codelet_cooperative(xs, 32) == g["sum"][0]
    # min/max through the cooperative tree with identity padding (reading R5)
    assert pc.codelet_cooperative(xs, 32, op=min, ident=I32_MAX) == g["min"][0]
    assert pc.codelet_cooperative(xs, 32, op=max, ident=I32_MIN) == g["max"][0]


# ------------------------------------------------------------ codelet replays
@pytest.mark.parametrize("seed", range(5))
def test_codelets_reach_plain_definition(seed):
    rnd = random.Random(seed)
    n = rnd.randint(0, 3000)
    xs = [rnd.randint(-1000, 1000) for _ in range(n)]
    want = int(oracle.reduce(np.array(xs, np.int32), "sum").value)
    assert pc.codelet_scalar(xs) == want
    for p in (1, 3, 64):
        for pat in ("tiled", "strided"):
            for comb in ("spectrum", "atomic"):
                assert pc.codelet_compound(xs, p, pat, comb) == want
    assert pc.codelet_cooperative(xs, 32) == want
    assert pc.codelet_va1(xs) == want
    assert pc.codelet_va2(xs, 32) == want
    if n:
        assert pc.codelet_cooperative(xs, 32, op=min, ident=I32_MAX) == int(oracle.reduce(np.array(xs, np.int32), "min").value)


# ------------------------------------------------------------ P8 brute force vs exact ref
@pytest.mark.parametrize("dtype", ["int32", "float32", "float64"])
@pytest.mark.parametrize("dist", ["uniform01", "uniform_pm1", "int_full", "int_small"])
def test_p8_oracle_vs_exact_ref(dtype, dist):
    for k, n in enumerate([0, 1, 2, 31, 32, 33, 1000, 4097]):
        x = synth.make(dtype, n, dist, 100 * k + 7)
        if dtype == "int32":
            assert int(oracle.reduce(x, "sum").value) == ref.sum_i32(x)
            assert int(oracle.reduce(x, "min").value) == ref.min_i32(x)
            assert int(oracle.reduce(x, "max").value) == ref.max_i32(x)
        else:
            w = 32 if dtype == "float32" else 64
            r = oracle.reduce(x, "sum")
            exact = ref.sum_fp(x)
            # Neumaier in double: |S - exact| <= 2 u_d |S| + n u_d^2 A
            assert abs(r.value - exact) <= oracle.oracle_error_bound(r, x.dtype, n), (n, r.value, exact)
            assert r.abs_sum == pytest.approx(ref.abs_sum(x), rel=n * 2.0 ** -52 + 1e-300)
            assert oracle.reduce(x, "min").bits == ref.minmax_fp_bits(x, "min", w)
            assert oracle.reduce(x, "max").bits == ref.minmax_fp_bits(x, "max", w)


def test_compensation_catches_cancellation():
    # naive double summation gives 0.0 here; the exact (and Neumaier) answer is 2.0
    x = np.array([1e16, 1.0, -1e16, 1.0], np.float64)
    naive = 0.0
    for v in x:  # plain left-to-right double loop (Python 3.12's sum() is compensated)
        naive = naive + float(v)
    assert naive != 2.0
    assert oracle.reduce(x, "sum").value == 2.0 == ref.sum_fp(x)


# ------------------------------------------------------------ P11 special values
@pytest.mark.parametrize("dtype", ["float32", "float64"])
def test_p11_special_values(dtype):
    sp = lambda k: synth.special_f(dtype, k)
    dt = synth.NP_DTYPE[dtype]
    nanbits = oracle.CANONICAL_NAN32 if dtype == "float32" else oracle.CANONICAL_NAN64
    bits = f32bits if dtype == "float32" else f64bits
    base = np.array([1.0, -2.0, 3.0, 0.5], dt)
    for kind in ("nan", "neg_nan"):
        x = base.copy(); x[2] = sp(kind)
        assert math.isnan(oracle.reduce(x, "sum").value)
        assert oracle.reduce(x, "min").bits == nanbits
        assert oracle.reduce(x, "max").bits == nanbits
    x = base.copy(); x[1] = sp("inf")
    assert oracle.reduce(x, "sum").value == math.inf
    assert oracle.reduce(x, "max").bits == bits(math.inf)
    x[3] = sp("ninf")
    assert math.isnan(oracle.reduce(x, "sum").value)
    assert oracle.reduce(x, "min").bits == bits(-math.inf)
    # signed zeros: -0.0 < +0.0, regardless of order
    for arr in ([0.0, -0.0], [-0.0, 0.0], [-0.0, -0.0, 0.0, -0.0]):
        x = np.array(arr, dt)
        assert oracle.reduce(x, "min").bits == bits(-0.0)
        assert oracle.reduce(x, "max").bits == bits(0.0)
    x = np.array([-0.0, -0.0], dt)
    assert oracle.reduce(x, "max").bits == bits(-0.0)
    # all-NaN, n = 1
    x = np.full(5, sp("nan"), dt)
    assert oracle.reduce(x, "max").bits == nanbits
    x = np.array([-3.25], dt)
    assert oracle.reduce(x, "min").value == -3.25 and oracle.reduce(x, "sum").value == -3.25


def test_p11_empty_identities():
    e32, ef, ed = np.zeros(0, np.int32), np.zeros(0, np.float32), np.zeros(0, np.float64)
    assert oracle.reduce(e32, "sum").value == 0
    assert oracle.reduce(e32, "min").value == I32_MAX
    assert oracle.reduce(e32, "max").value == I32_MIN
    assert oracle.reduce(ef, "sum").value == 0.0
    assert oracle.reduce(ef, "min").bits == f32bits(math.inf)
    assert oracle.reduce(ef, "max").bits == f32bits(-math.inf)
    assert oracle.reduce(ed, "min").bits == f64bits(math.inf)
    assert oracle.reduce(ed, "max").bits == f64bits(-math.inf)


# ------------------------------------------------------------ gates detect mistakes
@pytest.mark.parametrize("dtype", ["float32", "float64"])
def test_gates_reject_dropped_or_duplicated_element(dtype):
    n = 1 << 12
    x = synth.make(dtype, n, "uniform01", 3)
    r = oracle.reduce(x, "sum")
    good = float(np.sum(x.astype(np.float64)))
    ok, _ = oracle.check_sum(good, r, x.dtype, n, chain=64)
    assert ok
    for bad in (good - float(x[17]), good + float(x[5]), -good):
        ok, msg = oracle.check_sum(bad, r, x.dtype, n, chain=64)
        assert not ok, msg


def test_omp_baseline_runs():
    x = synth.make("float32", 1 << 16, "ones", 0)
    assert oracle.omp_sum_f32(x) == float(1 << 16)
    assert oracle.omp_threads() >= 1


# ------------------------------------------------------------ histogram (N4)
def test_histogram_closed_forms():
    # iota over [0, 1024) into 16 bins: 64 each; out-of-range values not counted
    x = np.arange(-100, 1124, dtype=np.int32)
    c = oracle.histogram(x, 0, 1024, 16)
    assert c.tolist() == [64] * 16
    assert oracle.histogram(np.ones(1000, np.int32), 0, 10, 10).tolist() == [0, 1000] + [0] * 8
    assert oracle.histogram(np.zeros(0, np.int32), 0, 10, 3).tolist() == [0, 0, 0]
    f = np.array([np.nan, np.inf, -np.inf, 0.5, 0.25, 0.999, 1.0, -0.0], np.float32)
    assert oracle.histogram(f, 0.0, 1.0, 4).tolist() == [1, 1, 1, 1]  # -0.0 is in [0, 1)


@pytest.mark.parametrize("dtype", ["int32", "float32"])
@pytest.mark.parametrize("nbins", [1, 7, 64, 1000])
def test_histogram_vs_exact_rational(dtype, nbins):
    rng = np.random.Generator(np.random.PCG64(nbins))
    if dtype == "int32":
        x = rng.integers(-50, 5000, 3000).astype(np.int32)
        lo, hi = 0, 4096  # power-of-two range: every edge is exact
    else:
        x = (rng.random(3000, dtype=np.float32) * 2 - 0.5).astype(np.float32)
        lo, hi = 0.0, 1.0
    c = oracle.histogram(x, lo, hi, nbins)
    want = ref.histogram(x, lo, hi, nbins)
    if dtype == "int32" or nbins in (1, 64):  # exact integer rule / power-of-two fp32 grid: no rounding
        assert c.tolist() == want
    assert int(c.sum()) == sum(want) == int(((x >= lo) & (x < hi)).sum())
    assert np.abs(c.astype(np.int64) - np.array(want)).sum() <= 2 * max(1, nbins // 100) + 2


def _edge_distance_bound(p, lo, hi, nbins):
    """Largest shift, in bin units, that the fp32 rule's roundings can give the
    position p = (x - lo) * nbins / (hi - lo): lo_f = fl32(lo) moves the origin
    by <= u|lo|, scale = fl32(nbins / (hi - lo)) is off by <= u * scale, and
    fl32(x - lo_f), fl32(d * scale) each add <= u of their result (u = 2^-24);
    doubled for slack in the products."""
    u = 2.0 ** -24
    scale = nbins / (hi - lo)
    return 2 * (3 * u * (abs(p) + 1) + u * abs(lo) * scale) + 2.0 ** -40


@pytest.mark.parametrize("lo,hi,nbins", [(0.0, 1.0, 7), (0.0, 1.0, 1000), (-3.7, 11.3, 257),
                                         (0.1, 0.7, 100), (-1.0, 1.0, 65535), (1000.0, 1000.5, 3),
                                         (-2.0 ** 20, 3.0, 12345)])
def test_histogram_f32_rule_vs_exact_rational_per_element(lo, hi, nbins):
    """oracle_histogram_f32 off power-of-two grids: its bin
    rule floor(fl32(fl32(x - lo_f) * scale)) is a definition chosen for the
    kernel (DESIGN R13), so it is pinned here against the exact-rational
    definition floor((x - lo) * nbins / (hi - lo)) of oracle/ref.py element by
    element: every element where the two disagree must sit within the fp32
    rule's rounding reach of an integer bin edge (0, ..., nbins), and nowhere
    else.  Inputs mix uniform values with values planted on both sides of
    every kind of edge (the first few, some interior ones, lo and hi), so the
    disagreements actually occur."""
    from fractions import Fraction
    rng = np.random.Generator(np.random.PCG64(nbins))
    width = hi - lo
    xs = list((lo - 0.05 * width + rng.random(1500) * 1.1 * width).astype(np.float32))
    edges = list(range(0, min(nbins, 40) + 1)) + list(rng.integers(0, nbins + 1, 40)) + [nbins]
    for k in edges:
        e = np.float32(lo + width * int(k) / nbins)
        for step in range(-3, 4):
            v = e
            for _ in range(abs(step)):
                v = np.nextafter(v, np.float32(np.inf if step > 0 else -np.inf), dtype=np.float32)
            xs.append(np.float32(v))
    x = np.array(xs, np.float32)
    flo, fw = Fraction(lo), Fraction(hi) - Fraction(lo)
    disagree = 0
    for v in x:
        c = oracle.histogram(np.array([v], np.float32), lo, hi, nbins)
        got = int(np.flatnonzero(c)[0]) if c.any() else None
        p = (Fraction(float(v)) - flo) * nbins / fw
        want = int(p // 1) if 0 <= p < nbins else None
        if got == want:
            continue
        disagree += 1
        dist = abs(float(p - round(p)))
        assert dist <= _edge_distance_bound(float(p), lo, hi, nbins), (float(v), got, want, float(p), dist)
        # a rounding moves x by at most one bin, never further
        assert got is None or want is None or abs(got - want) == 1, (float(v), got, want)
    assert disagree <= len(x) // 4
    # the whole-array counts: the same totals up to the edge elements
    c = oracle.histogram(x, lo, hi, nbins)
    want = ref.histogram(x, lo, hi, nbins)
    assert np.abs(c.astype(np.int64) - np.array(want)).sum() <= 2 * disagree


def test_histogram_f32_rule_disagreements_exist():
    """The per-element pin above is not vacuous: on a non-power-of-two grid
    with points planted at the edges, the fp32 rule and the exact-rational rule
    do disagree somewhere (else the pin would pass a kernel that used either)."""
    from fractions import Fraction
    lo, hi, nbins = 0.1, 0.7, 100
    n_dis = 0
    for k in range(nbins + 1):
        e = np.float32(lo + (hi - lo) * k / nbins)
        for v in (np.nextafter(e, np.float32(-1), dtype=np.float32), e, np.nextafter(e, np.float32(2), dtype=np.float32)):
            c = oracle.histogram(np.array([v], np.float32), lo, hi, nbins)
            got = int(np.flatnonzero(c)[0]) if c.any() else None
            p = (Fraction(float(v)) - Fraction(lo)) * nbins / (Fraction(hi) - Fraction(lo))
            want = int(p // 1) if 0 <= p < nbins else None
            n_dis += got != want
    assert n_dis > 0
