"""The test-side chain bound L of gate G2 (tests/_chain.py) on CPU: the
library's own plan["chain"] is never below it, over every auto-dispatched size
and every forced variant the GPU tests run; and hand-counted values for a few
launch shapes, so a slip in the formula itself fails here."""
import itertools

import pytest

import paper_conf_cgo_gonzalohghmh19_b200 as rb
from tests._chain import chain_bound, checked_chain

VARIANTS = [dict(), dict(mode="deterministic"), dict(grid_combine=0, block=256), dict(grid_combine=1),
            dict(grid_combine=2), dict(grid_combine=3), dict(grid_combine=4, grid=16),
            dict(stage="smem", unroll=8, block=256), dict(stage="smem", unroll=16, block=256),
            dict(block_combine=3, block=128), dict(block_combine=1), dict(block_combine=2, block=128),
            dict(grid=148, grid_combine=3), dict(grid=148, grid_combine=1, unroll=1),
            dict(grid=7, grid_combine=2, block=64, unroll=2), dict(grid_combine=5), dict(grid_combine=5, block=32, unroll=1),
            dict(grid=300, grid_combine=5, block=128), dict(input_ready=True), dict(input_ready=True, mode="deterministic")]


@pytest.mark.parametrize("dtype,op", [("float32", "sum"), ("float64", "sum"), ("float32", "sum_accurate"),
                                      ("float64", "sum_accurate")])
def test_library_chain_never_below_test_bound(dtype, op):
    sizes = [0, 1, 7, 255, 4097, 65537, (1 << 20) + 3, 1 << 24, 1 << 26, 1 << 28, 1 << 31]
    checked = 0
    for n, v in itertools.product(sizes, VARIANTS):
        if op == "sum_accurate" and dtype == "float64" and (v.get("grid_combine") == 1 or
                                                            v.get("block_combine") in (1, 2)):
            continue  # rejected combos (no double-double atomics)
        if v.get("mode") == "deterministic" and v.get("grid_combine") == 1:
            continue
        for align in (0, 4, 12):
            try:
                p = rb.query_plan(dtype, op, n, in_ptr=4096 + align * (2 if dtype == "float64" else 1), **v)
            except rb.ReduceError:
                continue
            checked_chain(dtype, op, p)
            checked += 1
    assert checked > 300


def test_exact_ops_have_no_chain():
    for dt, op in (("int32", "sum"), ("int32", "max"), ("float32", "min"), ("float64", "max")):
        assert chain_bound(dt, op, rb.query_plan(dt, op, 1 << 20)) == 0


def _plan(**kw):
    base = dict(grid=1, block=256, unroll=4, tiles=1, slots=0, grid_combine=0, block_combine=0, chain=0)
    base.update(kw)
    return base


def test_hand_counted_chains():
    # headline shape: 2^28 fp32, 32768 blocks x 256 threads x 4 vectors, ATOMIC, Vs.
    # thread: 2 vectors per accumulator + 3 (8-lane tree) + 1 (head/tail) + 1 (merge) = 7;
    # block: 5 + 5; fp32 -> one final rounding: 18
    p = _plan(grid=32768, block=256, unroll=4, tiles=32768, slots=32, grid_combine=1)
    assert chain_bound("float32", "sum", p) == 18
    # the same in fp64 (4-lane tree: 2): 2 + 2 + 2 = 6 thread, 10 block, 32768/32 + 5 grid
    assert chain_bound("float64", "sum", p) == 6 + 10 + 1024 + 5
    # fp64 TWO_PASS with 1000 blocks: ceil(1000 / 1024) + 2 + 5 + 5 = 13 above the block
    p = _plan(grid=1000, block=512, unroll=2, tiles=3000, grid_combine=2)
    assert chain_bound("float64", "sum", p) == (1 * 3 + 4) + 10 + 13
    # single block, one warp, U = 1, fp32: 5 tiles -> 5 vectors on accumulator 0,
    # + 3 + 2, a 5-level warp butterfly, no second butterfly, no rounding
    p = _plan(grid=1, block=32, unroll=1, tiles=5, grid_combine=0)
    assert chain_bound("float32", "sum", p) == 5 + 3 + 2 + 5
    # the same with VA1 (fp64 shared accumulator): + one fp32 rounding
    assert chain_bound("float32", "sum", dict(p, block_combine=2)) == 5 + 3 + 2 + 0 + 1
    # fp64 VA1 in a 128-thread block: 128 shared additions
    assert chain_bound("float64", "sum", dict(p, block=128, block_combine=2)) == 5 + 2 + 2 + 128
    # accurate fp32, 3 tiles per block of U = 8: 24 lane additions + 1 + 3 (8 accumulators)
    p = _plan(grid=10, block=256, unroll=8, tiles=30, grid_combine=4)
    assert chain_bound("float32", "sum_accurate", p) == 24 + 1 + 3 + 10 + 5
    # fp64 FLAGS, 2000 blocks of 256: the polling thread folds ceil(2000/256) = 8
    # records, then two 5-level butterflies
    p = _plan(grid=2000, block=256, unroll=4, tiles=2000, grid_combine=5)
    assert chain_bound("float64", "sum", p) == (2 + 2 + 2) + 10 + 8 + 10
    # empty input: only the fixed levels remain
    assert chain_bound("float32", "sum", _plan(tiles=0)) == 0 + 3 + 2 + 10
