"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element
by element on the same seeded inputs.  Integer and min/max results must be
bit-exact; fp sums must pass gate G1 (north star) and the tight gate G2
(chain-length bound of the variant that ran).  Pins P1-P11 of DESIGN.md."""
import math

import numpy as np
import pytest

import oracle
import synth
from tests._util import check, gpu_reduce_many, to_device, NP

pytestmark = pytest.mark.gpu

DTYPES = ["int32", "float32", "float64"]
OPS = ["sum", "min", "max"]


def _rb():
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    return rb


def _dist(dtype):
    return "int_full" if dtype == "int32" else "uniform_pm1"


# ------------------------------------------------------------- P6 / P7 paper examples
@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("variant", [dict(), dict(block=32, grid_combine=0), dict(block=256, unroll=1, grid_combine=1),
                                     dict(block=32, unroll=1, grid_combine=2), dict(block=64, grid_combine=3)])
def test_p6_fig1c_example_and_p7_fig2(dtype, variant):
    for xs, want in ((list(range(16)), 120), (list(range(1, 35)), 595)):
        x = np.array(xs, NP[dtype])
        for off in range(4):
            t = to_device(x, off)
            (got,), (plan,) = gpu_reduce_many([(t, "sum")], **variant)
            assert got[0] == want
            (mn,), _ = gpu_reduce_many([(t, "min")], **variant)
            (mx,), _ = gpu_reduce_many([(t, "max")], **variant)
            assert mn[0] == xs[0] and mx[0] == xs[-1]


# ------------------------------------------------------------- P8 brute force, small n
SMALL_N = sorted(set(list(range(0, 130)) + [255, 256, 257, 511, 512, 513, 1023, 1024, 1025, 2047, 2048, 2049,
                                             4095, 4096, 4097, 8191, 8193, 16385, 65535, 65536, 65537]))


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("mode", ["fast", "deterministic"])
def test_p8_small_sizes_all_offsets(dtype, mode):
    cases, xs = [], []
    for k, n in enumerate(SMALL_N):
        x = synth.make(dtype, n, _dist(dtype), 1000 + k)
        for off in range(8 if dtype != "float64" else 4):
            t = to_device(x, off)
            for op in OPS:
                cases.append((t, op))
                xs.append((x, op))
    got, plans = gpu_reduce_many(cases, mode=mode)
    for (x, op), g, p in zip(xs, got, plans):
        check(x, op, g, p)


# ------------------------------------------------------------- P1 / P2 / P3 closed forms on the GPU
@pytest.mark.parametrize("n", [1000, 4097, (1 << 20) + 3, (1 << 24)])
def test_p1_ones_and_p2_iota(n):
    rb = _rb()
    import torch
    for dtype in DTYPES:
        t = torch.ones(n, dtype=getattr(torch, dtype), device="cuda")
        assert rb.reduce(t, "sum").item() == n
        it = torch.arange(n, dtype=torch.int64, device="cuda").to(getattr(torch, dtype))
        r = rb.reduce(it, "sum").item()
        exact = n * (n - 1) // 2
        if dtype == "int32":
            exact = ((exact + 2 ** 31) % 2 ** 32) - 2 ** 31
            assert r == exact
        elif dtype == "float64":
            assert r == exact  # exact for n <= 2^27
        assert rb.reduce(it, "min").item() == 0 and rb.reduce(it, "max").item() == n - 1


@pytest.mark.parametrize("dtype,bound,n", [("float32", 1 << 7, (1 << 17) - 3), ("float64", 1 << 20, (1 << 22) + 5)])
def test_p3_integer_valued_sums_bit_exact(dtype, bound, n):
    x = synth.make(dtype, n, "intvalued", 77, bound=bound)
    exact = int(x.astype(np.int64).sum())
    for mode in ("fast", "deterministic"):
        (g,), _ = gpu_reduce_many([(to_device(x, 1), "sum")], mode=mode)
        assert float(g[0]) == exact


# ------------------------------------------------------------- sweep 2^k-1, 2^k, 2^k+1
@pytest.mark.parametrize("dtype", DTYPES)
def test_size_sweep(dtype):
    cases, xs = [], []
    for k in range(10, 25, 2):
        for d in (-1, 0, 1):
            n = (1 << k) + d
            x = synth.make(dtype, n, "uniform01" if dtype != "int32" else "int_full", 50 + k)
            t = to_device(x, (k + d) % 3)
            for op in OPS:
                cases.append((t, op))
                xs.append((x, op))
    for mode in ("fast", "deterministic"):
        got, plans = gpu_reduce_many(cases, mode=mode)
        for (x, op), g, p in zip(xs, got, plans):
            check(x, op, g, p)


# ------------------------------------------------------------- every variant on the same inputs
VARIANTS = []
for bc in range(4):
    for gc in range(6):
        for blk, u, st in ((32, 1, 1), (128, 2, 1), (256, 4, 1), (512, 8, 1), (1024, 1, 1),
                           (32, 16, 2), (128, 16, 2), (256, 8, 2), (1024, 4, 2)):
            VARIANTS.append(dict(block_combine=bc, grid_combine=gc, block=blk, unroll=u, stage=st))


@pytest.mark.parametrize("dtype", DTYPES)
def test_every_variant(dtype):
    n = (1 << 18) + 13
    x = synth.make(dtype, n, _dist(dtype), 4242)
    x[[0, n // 2, n - 1]] = x[[n - 1, 0, n // 2]]
    t = to_device(x, 3)
    for v in VARIANTS:
        if dtype == "float64" and v["block"] > 512 and v["unroll"] >= 2 and v["stage"] == 1:
            continue
        got, plans = gpu_reduce_many([(t, op) for op in OPS], **v)
        for op, g, p in zip(OPS, got, plans):
            check(x, op, g, p)


@pytest.mark.parametrize("dtype", DTYPES)
def test_cluster_dsmem_combine_all_sizes(dtype):
    """GC_CLUSTER: one cluster of C CTAs (C = 1..16) combining through DSMEM;
    deterministic (no atomics) and exact for int32 / min / max."""
    cases, xs, plans_kw = [], [], []
    for k, n in enumerate([1, 33, 4097, 65537, (1 << 20) + 3]):
        x = synth.make(dtype, n, _dist(dtype), 300 + k)
        t = to_device(x, k % 4)
        for C in (1, 2, 3, 8, 13, 16):
            for blk in (128, 512):
                got, plans = gpu_reduce_many([(t, op) for op in OPS], grid_combine=4, grid=C, block=blk)
                for op, g, p in zip(OPS, got, plans):
                    check(x, op, g, p)
                    assert p["grid_combine"] == 4 and p["grid"] <= C


@pytest.mark.parametrize("grid", [1, 7, 148, 1000])
def test_persistent_grids(grid):
    """Blocks looping over tiles (grid < tiles): the Catanzaro-style persistent
    partition must cover every tile exactly once."""
    for dtype in DTYPES:
        x = synth.make(dtype, (1 << 20) + 5, _dist(dtype), grid)
        t = to_device(x, 1)
        for gc, st in ((1, 1), (2, 1), (3, 1), (1, 2), (2, 2)):
            got, plans = gpu_reduce_many([(t, op) for op in OPS], grid=grid, grid_combine=gc, stage=st)
            for op, g, p in zip(OPS, got, plans):
                check(x, op, g, p)


# ------------------------------------------------------------- P5 permutations: extremes everywhere
@pytest.mark.parametrize("dtype", DTYPES)
def test_p5_permutation_extremes_in_head_tail_and_boundaries(dtype):
    rb = _rb()
    n = 100003
    base = synth.make(dtype, n, "perm", 9)
    plan = rb.query_plan(dtype, "min", n, in_ptr=0x1008)
    tile = plan["block"] * plan["unroll"] * (8 if dtype != "float64" else 4)
    positions = [0, 1, 2, n - 1, n - 2, tile - 1, tile, tile + 1, n // 2]
    for pos in positions:
        x = base.copy()
        i0, i1 = int(np.where(x == 0)[0][0]), int(np.where(x == n - 1)[0][0])
        x[[i0, pos]] = x[[pos, i0]]
        got, plans = gpu_reduce_many([(to_device(x, 1), "min"), (to_device(x, 1), "max")])
        assert got[0][0] == 0 and got[1][0] == n - 1


# ------------------------------------------------------------- P11 special values
@pytest.mark.parametrize("dtype", ["float32", "float64"])
@pytest.mark.parametrize("variant", [dict(), dict(mode="deterministic"), dict(block=32, grid_combine=0),
                                     dict(block_combine=1), dict(block_combine=2), dict(block_combine=3),
                                     dict(grid_combine=3)])
def test_p11_special_values(dtype, variant):
    dt = NP[dtype]
    n = 50000
    sp = lambda k: synth.special_f(dtype, k)
    cases = []
    for where in (0, 7, 24999, n - 1):
        for kind in ("nan", "neg_nan", "inf", "ninf"):
            x = synth.make(dtype, n, "uniform_pm1", 5)
            x[where] = sp(kind)
            cases.append(x)
        x = synth.make(dtype, n, "uniform_pm1", 6)
        x[where] = sp("inf"); x[(where + 11) % n] = sp("ninf")
        cases.append(x)
    # signed zeros
    z = np.zeros(n, dt); z[::3] = -0.0
    cases.append(z)
    cases.append(np.full(n, -0.0, dt))
    cases.append(np.full(n, sp("nan"), dt))
    cases.append(np.array([-0.0, 0.0] * 20, dt))
    for x in cases:
        t = to_device(x, 2)
        got, plans = gpu_reduce_many([(t, op) for op in OPS], **variant)
        for op, g, p in zip(OPS, got, plans):
            check(x, op, g, p)


def test_p11_empty_and_single():
    rb = _rb()
    import torch
    for dtype in DTYPES:
        e = torch.empty(0, dtype=getattr(torch, dtype), device="cuda")
        for op in OPS:
            got = rb.reduce(e, op).cpu().numpy()
            check(np.zeros(0, NP[dtype]), op, got)
        one = torch.tensor([-3], dtype=getattr(torch, dtype), device="cuda")
        for op in OPS:
            assert rb.reduce(one, op).item() == -3


# ------------------------------------------------------------- P9 determinism / invariants
@pytest.mark.parametrize("dtype", ["float32", "float64"])
@pytest.mark.parametrize("gc", [2, 3])
def test_p9_deterministic_mode_bitwise_repeatable(dtype, gc):
    import torch
    rb = _rb()
    x = synth.make(dtype, (1 << 22) + 77, "uniform_pm1", 31)
    t = to_device(x, 1)
    outs = torch.empty(100, dtype=t.dtype, device="cuda")
    for i in range(100):
        rb.reduce(t, "sum", out=outs[i:i + 1], mode="deterministic", grid_combine=gc)
    o = outs.cpu().numpy()
    assert len(set(o.view(np.uint32 if dtype == "float32" else np.uint64).tolist())) == 1
    check(x, "sum", o[:1], rb.query_plan(dtype, "sum", x.size, in_ptr=t.data_ptr(), mode="deterministic", grid_combine=gc))


def test_p9_int_results_permutation_invariant():
    rb = _rb()
    x = synth.make("int32", (1 << 20) + 9, "int_full", 8)
    rng = np.random.Generator(np.random.PCG64(1))
    y = rng.permutation(x)
    got, _ = gpu_reduce_many([(to_device(x), op) for op in OPS] + [(to_device(y, 5), op) for op in OPS])
    assert [int(g[0]) for g in got[:3]] == [int(g[0]) for g in got[3:]]


# ------------------------------------------------------------- full sizes (bench launch config)
def test_full_size_fp32_sum_2p28_bench_config():
    """BASELINE configs[1] at its largest point (2^28 fp32) in the exact launch
    configuration bench.py times (default dispatch, fast mode), whole-array
    oracle comparison with G1 and G2; plus deterministic mode."""
    rb = _rb()
    n = 1 << 28
    x = synth.make("float32", n, "uniform01", synth.seed_for(1, n))
    t = to_device(x)
    for mode in ("fast", "deterministic"):
        (g,), (p,) = gpu_reduce_many([(t, "sum")], mode=mode)
        check(x, "sum", g, p)
    xm = synth.make("float32", n, "uniform_pm1", synth.seed_for(1, n) + 1)
    tm = to_device(xm)
    got, plans = gpu_reduce_many([(tm, op) for op in OPS])
    for op, g, p in zip(OPS, got, plans):
        check(xm, op, g, p)


def test_full_size_int32_and_fp64_2p26_config3():
    """BASELINE configs[2]: int32 / fp64 sum, min, max at 64M elements, atomic
    vs deterministic-tree variants; int32 full range with INT32_MIN/MAX planted
    (one in the tail), fp64 integer-valued (exact, P3) with +-2.0 planted."""
    n = 1 << 26
    xi = synth.make("int32", n, "int_full", synth.seed_for(2, n))
    synth.plant(xi, [np.iinfo(np.int32).min, np.iinfo(np.int32).max], seed=3, positions=[12345, n - 3])
    xd = synth.make("float64", n, "intvalued", synth.seed_for(2, n) + 1, bound=1 << 20)
    synth.plant(xd, [2.0 ** 21, -(2.0 ** 21)], seed=4, positions=[n - 1, 777])
    for x in (xi, xd):
        t = to_device(x, 1)
        for mode in ("fast", "deterministic"):
            got, plans = gpu_reduce_many([(t, op) for op in OPS], mode=mode)
            for op, g, p in zip(OPS, got, plans):
                check(x, op, g, p)
            if x.dtype == np.float64:
                assert float(got[0][0]) == float(int(x.astype(np.int64).sum()))  # P3 bit-exact


def test_full_size_2p31_elements_64bit_indexing():
    """BASELINE configs[4] at k=1: 2^31 fp32 (8 GiB) on one GPU.  Property pins
    at full size: sum of ones is exactly 2^31 (every 8192-element tile sum is
    exact in fp32 and blocks combine exactly in fp64), int32 ones wrap to
    INT32_MIN, and a planted extreme at the very end is found."""
    import torch
    rb = _rb()
    n = 1 << 31
    t = torch.ones(n, dtype=torch.float32, device="cuda")
    assert rb.reduce(t, "sum").item() == float(n)
    assert rb.reduce(t, "sum", mode="deterministic").item() == float(n)
    t[n - 1] = 5.0
    t[3] = -7.0
    assert rb.reduce(t, "max").item() == 5.0 and rb.reduce(t, "min").item() == -7.0
    del t
    torch.cuda.empty_cache()
    ti = torch.ones(n, dtype=torch.int32, device="cuda")
    assert rb.reduce(ti, "sum").item() == -(2 ** 31)
    del ti
    torch.cuda.empty_cache()


# ------------------------------------------------------------- workspace / graphs / streams
def test_graph_capture_after_prepare():
    import torch
    rb = _rb()
    x = synth.make("float32", (1 << 22) + 3, "uniform01", 2)
    t = to_device(x, 1)
    s = torch.cuda.Stream()
    out = torch.empty(1, dtype=torch.float32, device="cuda")
    with torch.cuda.stream(s):
        # not prepared: capture must fail cleanly with NOT_PREPARED
        g = torch.cuda.CUDAGraph()
        with pytest.raises(Exception):
            with torch.cuda.graph(g, stream=s):
                rb.reduce(t, "sum", out=out, mode="deterministic")
    s2 = torch.cuda.Stream()
    rb.prepare(s2, t.numel())
    g2 = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g2, stream=s2):
        rb.reduce(t, "sum", out=out, stream=s2)
    for _ in range(3):
        out.zero_()
        g2.replay()
        torch.cuda.synchronize()
        check(x, "sum", out.cpu().numpy(), rb.query_plan("float32", "sum", t.numel(), in_ptr=t.data_ptr()))


def test_concurrent_streams_private_workspaces():
    import torch
    rb = _rb()
    xs = [synth.make("float64", (1 << 20) + i, "uniform01", i) for i in range(4)]
    ts = [to_device(x, i) for i, x in enumerate(xs)]
    streams = [torch.cuda.Stream() for _ in xs]
    outs = [torch.empty(1, dtype=torch.float64, device="cuda") for _ in xs]
    for _ in range(20):
        for t, s, o in zip(ts, streams, outs):
            rb.reduce(t, "sum", out=o, stream=s)
    torch.cuda.synchronize()
    for x, o, t in zip(xs, outs, ts):
        check(x, "sum", o.cpu().numpy(), rb.query_plan("float64", "sum", t.numel(), in_ptr=t.data_ptr()))


# ------------------------------------------------------------- end-to-end host entry
@pytest.mark.parametrize("dtype", DTYPES)
def test_reduce_host_chunks(dtype):
    import torch
    rb = _rb()
    n = (1 << 24) + 1001  # several 32 MiB chunks for fp64, 2+ for 4-byte types
    x = synth.make(dtype, n, _dist(dtype), 12)
    pinned = torch.from_numpy(x).pin_memory()
    for op in OPS:
        for src in (pinned, x):
            g = rb.reduce_host(src, op)
            check(x, op, np.array([g], NP[dtype]), None, gates=("g1",))
    for op in OPS:
        g = rb.reduce_host(x[:0], op)
        check(x[:0], op, np.array([g], NP[dtype]))


def test_chained_calls_read_the_previous_output():
    """Chains of calls on one stream where a call reads the previous call's
    output (a reduce of the scalar just written; a reduce of a segmented
    output), back to back with distinct values every iteration.  (The host
    disables a kernel's early, pre-dependency loads when its input overlaps
    the last output, or after entry points whose outputs it does not track.)"""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    s = torch.cuda.Stream()
    rb.prepare(s, 1 << 20)
    n = 1 << 16
    xs = [torch.full((n,), float(k + 1), device="cuda") for k in range(64)]
    buf = torch.full((4,), float("-inf"), device="cuda")
    res = torch.empty(64, device="cuda")
    seg_out = torch.empty(8, device="cuda")
    res2 = torch.empty(64, device="cuda")
    offs = torch.arange(0, n + 1, n // 8, dtype=torch.int64, device="cuda")
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        for k in range(64):
            rb.reduce(xs[k], "sum", out=buf[0:1], stream=s)          # buf[0] = (k+1) * n
            rb.reduce(buf, "max", out=res[k:k + 1], stream=s)         # reads buf[0] just written
            rb.reduce_segmented(xs[k], offs, "sum", out=seg_out, stream=s)
            rb.reduce(seg_out, "sum", out=res2[k:k + 1], stream=s)    # reads the segmented output
    torch.cuda.synchronize()
    want = np.array([(k + 1) * n for k in range(64)], np.float32)
    assert (res.cpu().numpy() == want).all(), res.cpu().numpy()[:8]
    assert (res2.cpu().numpy() == want).all(), res2.cpu().numpy()[:8]


@pytest.mark.parametrize("tiles", [1, 2, 65534, 65535, 65536, 65537])
def test_int32_sum_packed_atomic_around_its_grid_limit(tiles):
    """int32 sums under the ATOMIC combine carry value and block count in one
    64-bit atomic word (count in bits 48-63, so grids below 2^16); 65536 blocks
    and up take the slots + ticket path.  Full-range values make every block
    carry into bits 32-47.  Back-to-back calls check the word is reset."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    n = tiles * 256 - 3  # 32 threads x 1 vector of 8 int32 per tile; a ragged tail
    x = synth.make("int32", n, "int_full", 77 + tiles)
    t = to_device(x)
    opts = dict(grid_combine=1, block=32, unroll=1, grid=-1)
    p = rb.query_plan("int32", "sum", n, in_ptr=t.data_ptr(), **opts)
    assert p["grid"] == tiles and p["grid_combine"] == 1
    outs = torch.empty(3, dtype=torch.int32, device="cuda")
    for i in range(3):
        rb.reduce(t, "sum", out=outs[i:i + 1], **opts)
    got = outs.cpu().numpy()
    want = oracle.reduce(x, "sum").bits
    assert all(int(g.view(np.uint32)) == want for g in got), (got, want)


def test_per_thread_default_streams_get_their_own_workspace():
    """cudaStreamPerThread has one handle value (0x2) in every host thread but
    names a different stream in each: concurrent ATOMIC calls from two threads
    must not share a workspace (tickets / accumulators), so the library keys
    workspaces by the CUDA stream id."""
    import threading
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    n = 1 << 20
    xs = [torch.full((n,), k + 1, dtype=torch.int32, device="cuda") for k in range(2)]
    outs = [torch.empty(400, dtype=torch.int32, device="cuda") for _ in range(2)]
    torch.cuda.synchronize()
    opts = rb.make_opts(grid_combine=1, block=256, unroll=1)
    errors = []

    def work(k):
        try:
            torch.cuda.set_device(0)
            for i in range(400):
                rb.reduce_ptr(rb.INT32, "sum", xs[k].data_ptr(), n, outs[k][i:i + 1].data_ptr(), 2, opts)
        except Exception as e:  # pragma: no cover
            errors.append(e)
    ts = [threading.Thread(target=work, args=(k,)) for k in range(2)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    torch.cuda.synchronize()
    assert not errors, errors
    for k in range(2):
        assert (outs[k].cpu().numpy() == (k + 1) * n).all(), k


def test_prepare_covers_the_widest_partials_grid():
    """reduce_prepare(stream, n) must size the partials for any plan of up to n
    elements: fp64 accurate sums carry 16-byte
    double-double partials, and fp64's smallest tile is 32 threads x 1 vector =
    128 elements, so a forced TWO_PASS / LAST_BLOCK grid of 32-thread blocks is
    the largest partials array.  Captured after prepare: no NOT_PREPARED."""
    import torch
    rb = _rb()
    n = 65536 * 128  # exactly kMaxPartialBlocks tiles of 128 fp64 elements
    x = synth.make("float64", n, "uniform_pm1", 12)
    t = to_device(x)
    s = torch.cuda.Stream()
    rb.prepare(s, n)
    outs = torch.empty(4, dtype=torch.float64, device="cuda")
    g = torch.cuda.CUDAGraph()
    variants = [dict(op="sum_accurate", grid_combine=2, block=32, unroll=1),
                dict(op="sum_accurate", grid_combine=3, block=32, unroll=1),
                dict(op="sum", grid_combine=2, block=32, unroll=1),
                dict(op="max", grid_combine=3, block=32, unroll=1, mode="deterministic")]
    with torch.cuda.graph(g, stream=s):
        for i, v in enumerate(variants):
            kw = {k: val for k, val in v.items() if k != "op"}
            rb.reduce(t, v["op"], out=outs[i:i + 1], stream=s, **kw)
    g.replay()
    torch.cuda.synchronize()
    for i, v in enumerate(variants):
        kw = {k: val for k, val in v.items() if k != "op"}
        p = rb.query_plan("float64", v["op"], n, in_ptr=t.data_ptr(), **kw)
        assert p["grid"] == 65536, p
        if v["op"] == "max":
            check(x, "max", outs[i:i + 1].cpu().numpy(), p)
        else:
            ref = oracle.reduce(x, "sum")
            assert abs(float(outs[i]) - ref.value) <= 2.0 ** -40 * ref.abs_sum, (v, float(outs[i]), ref.value)
