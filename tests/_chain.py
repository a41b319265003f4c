"""Test-side longest fp addition chain L of a reduction launch (gate G2).

G2 (reading R8): |r - S| <= (L + 1) u sum|x| for any
summation tree whose longest root-to-leaf path has L additions (Higham's
gamma_L bound).  L is computed HERE from the launch *shape* the plan reports
(grid, block, unroll, tiles, slots, grid / block combine, dtype, op) -- it is
never taken from the library's own ``plan["chain"]``, so a library that
over-counts its chain cannot loosen its own gate.  The tests assert
``plan["chain"] >= chain_bound(...)`` (the library's claim is not an
under-estimate) and gate on ``chain_bound``.

How each term follows from the partition the plan describes (DESIGN.md section 5,
the paper's Fig. 1(b) blocked / strided partition):
  * per thread: a block owns ceil(tiles / grid) tiles (tiles go to blocks with
    stride grid); in each tile a thread folds `unroll` 32-byte vectors.
      - plain sums: every vector is first reduced by a pairwise tree
        (log2(VE) levels, VE elements per vector), then added to one of TWO
        accumulators alternately -> ceil(unroll/2) additions per tile per
        accumulator; +1 for the head / tail element some threads fold into
        accumulator 0; +1 merging the two accumulators.
      - accurate sums: lane k of every vector goes to accumulator k (VE of
        them) -> unroll additions per tile; +1 head / tail; a pairwise tree over
        the VE accumulators (log2(VE) levels).
  * warp: a 5-level butterfly (32 lanes).
  * block: "Vs" (shared partial[32] then another 5-level butterfly when the
    block has more than one warp); "VA2+S" (a warp butterfly then one shared
    accumulator updated by each warp in turn: nw additions); "VA1" (every
    thread adds into one shared accumulator: block additions, no butterfly);
    "V" (a shared tree, log2(block) levels).  fp32 plain sums keep their block
    accumulator for VA2+S / VA1 in fp64 (the cross-block type), so those
    additions are counted in the fp64 term below instead.
  * grid: DIRECT none; CLUSTER <= 16 values in a 32-lane butterfly (5);
    ATOMIC: each of `slots` accumulators receives ceil(grid / slots) atomic
    additions, then a 32-lane butterfly (5); TWO_PASS / LAST_BLOCK: the
    partials are folded by one block of Bc threads into 4 accumulators per
    thread (stride Bc), joined (2), butterflied (5), the warps' values
    butterflied again (5).  Bc is at least 256 (TWO_PASS) or `block`
    (LAST_BLOCK); a smaller Bc only lengthens the chain, so Bc = 256 /
    block is an upper bound.  FLAGS: the polling block (`block` threads)
    folds the grid values into ONE accumulator per thread (stride block):
    ceil(grid / block) additions, butterflied (5), the warps' values
    butterflied again (5).
  * fp32 plain sums cross blocks in fp64: everything above the block adds
    < (grid + 64) 2^-53 sum|x|, which is < 2^-29 sum|x| = 1/32 u_f sum|x|
    for grid < 2^23, plus ONE fp32 rounding of the final value -> +1 (the
    DIRECT / single-block path with Vs or V converts a float to double and
    back exactly: +0).
"""
from __future__ import annotations

import math

VE = {"float32": 8, "float64": 4}   # elements per 32-byte vector
GC_DIRECT, GC_ATOMIC, GC_TWO_PASS, GC_LAST_BLOCK, GC_CLUSTER, GC_FLAGS = 0, 1, 2, 3, 4, 5
BC_SHFL, BC_ATOMIC_WARP, BC_ATOMIC_ALL, BC_TREE = 0, 1, 2, 3


def _cdiv(a: int, b: int) -> int:
    return -(-a // b)


def _grid_terms(gc: int, grid: int, block: int, slots: int) -> int:
    if gc == GC_DIRECT:
        return 0
    if gc == GC_CLUSTER:
        return 5
    if gc == GC_ATOMIC:
        return _cdiv(grid, max(1, slots)) + 5
    if gc == GC_FLAGS:
        return _cdiv(grid, block) + 5 + 5
    bc = 256 if gc == GC_TWO_PASS else block
    return _cdiv(grid, 4 * bc) + 2 + 5 + 5


def chain_bound(dtype: str, op: str, plan: dict) -> int:
    """Longest addition chain L of the launch `plan` describes (0 for exact ops)."""
    if dtype == "int32" or op not in ("sum", "sum_accurate"):
        return 0
    grid, block, unroll = plan["grid"], plan["block"], plan["unroll"]
    tiles, gc, bcomb = plan["tiles"], plan["grid_combine"], plan["block_combine"]
    ve = VE[dtype]
    tpb = _cdiv(tiles, grid) if tiles > 0 else 0
    nw = _cdiv(block, 32)
    lg_ve = int(math.log2(ve))
    if op == "sum":
        thread = _cdiv(unroll, 2) * tpb + lg_ve + 2
    else:
        thread = unroll * tpb + 1 + lg_ve
    fp32_plain = dtype == "float32" and op == "sum"
    if bcomb == BC_SHFL:
        blk = 5 + (5 if nw > 1 else 0)
    elif bcomb == BC_ATOMIC_WARP:
        blk = 5 + (0 if fp32_plain else nw)
    elif bcomb == BC_ATOMIC_ALL:
        blk = 0 if fp32_plain else block
    else:
        blk = int(math.log2(block))
    if fp32_plain:
        # one rounding of the fp64 block / grid value to fp32, except when a
        # single block's value never left fp32 (DIRECT with Vs or V)
        exact = gc == GC_DIRECT and bcomb in (BC_SHFL, BC_TREE)
        return thread + blk + (0 if exact else 1)
    return thread + blk + _grid_terms(gc, grid, block, plan["slots"])


def checked_chain(dtype: str, op: str, plan: dict) -> int:
    """chain_bound(), after asserting the library's own claim is not smaller."""
    L = chain_bound(dtype, op, plan)
    assert plan["chain"] >= L, f"library chain {plan['chain']} < test-side bound {L} for {dtype} {op} {plan}"
    return L
