"""GC_FLAGS (flag-in-data partial records polled by the last block, DESIGN.md
S5): parity against the oracle at every grid shape up to the 8192-block cap,
bitwise determinism, CUDA-graph replays (the epoch lives in device memory),
growth of the record area, independent streams, and the 32-bit epoch wrap."""
import os
import subprocess
import sys

import numpy as np
import pytest

import synth
from tests._util import BITS, check, gpu_reduce_many, to_device

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
DTYPES = ["int32", "float32", "float64"]
OPS = ["sum", "min", "max"]


def _rb():
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    return rb


def _dist(dtype):
    return "int_full" if dtype == "int32" else "uniform_pm1"


@pytest.mark.parametrize("dtype", DTYPES)
def test_flags_every_grid_shape(dtype):
    # grids 1, 2, 3, one less / one more than the poller's stride (block), a
    # ragged multiple, and the cap (8192 blocks, persistent tiles)
    cases = [((1 << 12) + 3, dict(block=32, unroll=1, grid=1)),
             ((1 << 12) + 3, dict(block=32, unroll=1, grid=2)),
             ((1 << 12) + 3, dict(block=32, unroll=1, grid=3)),
             ((1 << 16) + 7, dict(block=32, unroll=1, grid=31)),
             ((1 << 16) + 7, dict(block=32, unroll=1, grid=33)),
             ((1 << 18) + 13, dict(block=128, unroll=2, grid=-1)),
             ((1 << 20) + 5, dict(block=256, unroll=4, grid=-1)),
             ((1 << 22) + 1, dict(block=128, unroll=1, grid=-1)),   # 8192-block cap
             ((1 << 20) + 5, dict(block=1024, unroll=1, grid=600)),
             ((1 << 20) + 5, dict(stage="smem", block=256, unroll=8, grid=-1))]
    for i, (n, v) in enumerate(cases):
        x = synth.make(dtype, n, _dist(dtype), 900 + i)
        t = to_device(x, i % 3)
        for mode in ("fast", "deterministic"):
            got, plans = gpu_reduce_many([(t, op) for op in OPS], mode=mode, grid_combine=5, **v)
            for op, g, p in zip(OPS, got, plans):
                assert p["grid_combine"] == 5 and p["grid"] <= 8192
                check(x, op, g, p)


def test_flags_is_bitwise_deterministic():
    import torch
    rb = _rb()
    for dtype in ("float32", "float64"):
        x = synth.make(dtype, (1 << 22) + 11, "uniform_pm1", 77)
        t = to_device(x, 1)
        for op in ("sum", "sum_accurate"):
            outs = [rb.reduce(t, op, grid_combine=5, block=128, unroll=1) for _ in range(100)]
            torch.cuda.synchronize()
            bits = {int(o.cpu().numpy().view(BITS[dtype])[0]) for o in outs}
            assert len(bits) == 1, (dtype, op, bits)
            got = outs[0].cpu().numpy()
            if op == "sum":
                p = rb.query_plan(dtype, op, t.numel(), in_ptr=t.data_ptr(), grid_combine=5, block=128, unroll=1)
                check(x, op, got, p)


def test_flags_graph_replays_see_fresh_records():
    import torch
    rb = _rb()
    n = (1 << 21) + 3
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        rb.prepare(s, max_n=n)
        xs = [torch.zeros(n, dtype=torch.int32, device="cuda") for _ in range(3)]
        outs = [torch.empty(1, dtype=torch.int32, device="cuda") for _ in range(3)]
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for x, o in zip(xs, outs):
                rb.reduce(x, "sum", out=o, grid_combine=5, block=256, unroll=2)
    rng = np.random.default_rng(5)
    for rep in range(8):
        hs = [rng.integers(-1000, 1001, n, dtype=np.int32) for _ in range(3)]
        for x, h in zip(xs, hs):
            x.copy_(torch.from_numpy(h))
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        for o, h in zip(outs, hs):
            want = (int(h.astype(np.int64).sum()) + 2 ** 31) % 2 ** 32 - 2 ** 31  # int32 wrap-around sum
            assert int(o.item()) == want, (rep, int(o.item()), want)


def test_flags_record_area_grows_and_streams_are_independent():
    import torch
    rb = _rb()
    a = synth.make("float64", (1 << 23) + 9, "uniform_pm1", 31)
    b = synth.make("int32", (1 << 16) + 9, "int_full", 32)
    ta, tb = to_device(a, 0), to_device(b, 2)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    res = []
    for k in range(6):
        for s in (s1, s2):
            with torch.cuda.stream(s):
                # small grid, then a larger one (grows the stream's records), then small again
                grid = (7, 4000, 8192, 5, 8192, 1)[k]
                res.append(("max", a, rb.reduce(ta, "max", grid_combine=5, block=32, unroll=1, grid=grid)))
                res.append(("sum", b, rb.reduce(tb, "sum", grid_combine=5, block=32, unroll=1, grid=min(grid, 1000))))
    torch.cuda.synchronize()
    for op, x, o in res:
        check(x, op, o.cpu().numpy())


_WRAP = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import paper_conf_cgo_gonzalohghmh19_b200 as rb, oracle, synth
x = synth.make("int32", (1 << 18) + 5, "int_full", 3)
y = synth.make("float64", (1 << 18) + 5, "uniform_pm1", 4)
tx = torch.from_numpy(x).cuda(); ty = torch.from_numpy(y).cuda()
bad = 0
for i in range(12):   # epochs 0xFFFFFFFC .. wrap .. 8
    g = (300, 1000, 7, 2048)[i % 4]
    sx = rb.reduce(tx, "sum", grid_combine=5, block=32, unroll=1, grid=g)
    my = rb.reduce(ty, "max", grid_combine=5, block=32, unroll=1, grid=g)
    torch.cuda.synchronize()
    bad += int(sx.cpu().numpy().view(np.uint32)[0]) != oracle.reduce(x, "sum").bits
    bad += int(my.cpu().numpy().view(np.uint64)[0]) != oracle.reduce(y, "max").bits
print("BAD", bad)
"""


def test_flags_epoch_wrap():
    env = dict(os.environ, REDUCE_FLAGS_EPOCH0=str(0xFFFFFFFB))
    r = subprocess.run([sys.executable, "-c", _WRAP.format(root=ROOT)], env=env, capture_output=True, text=True,
                       timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "BAD 0" in r.stdout, r.stdout + r.stderr[-2000:]
