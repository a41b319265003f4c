"""Exact pure-Python reduction reference — TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Independent of ``oracle.c`` (no shared code): it pins the C oracle on small
inputs, using arithmetic that is exact by construction:

* int32 sum: Python big integers, then reduction modulo 2**32 into two's
  complement (reading R1 of DESIGN.md; the paper's ``int accum``).
* fp sum: ``math.fsum`` — the correctly rounded double of the exact real sum of
  the inputs (Shewchuk).  Non-finite inputs follow reading R2.
* min / max: comparison by an explicit total order in which -0.0 < +0.0 and any
  NaN wins (reading R3), result returned as a bit pattern.

Only for small n (pure-Python loops).
"""
from __future__ import annotations

import math
import struct

CANONICAL_NAN32 = 0x7FC00000
CANONICAL_NAN64 = 0x7FF8000000000000


def sum_i32(xs) -> int:
    s = sum(int(v) for v in xs) % (1 << 32)
    return s - (1 << 32) if s >= (1 << 31) else s


def min_i32(xs) -> int:
    return min((int(v) for v in xs), default=2 ** 31 - 1)


def max_i32(xs) -> int:
    return max((int(v) for v in xs), default=-(2 ** 31))


def sum_fp(xs) -> float:
    vals = [float(v) for v in xs]
    if any(math.isnan(v) for v in vals):
        return math.nan
    pinf = any(v == math.inf for v in vals)
    ninf = any(v == -math.inf for v in vals)
    if pinf and ninf:
        return math.nan
    if pinf:
        return math.inf
    if ninf:
        return -math.inf
    return math.fsum(vals)


def abs_sum(xs) -> float:
    return math.fsum(abs(float(v)) for v in xs if math.isfinite(float(v)))


def _rank(v: float):
    """Sort key of the total order R3 on non-NaN values: (value, sign bit flipped)."""
    return (v, 0 if math.copysign(1.0, v) < 0 else 1)


def _bits(v: float, width: int) -> int:
    if width == 32:
        return struct.unpack("<I", struct.pack("<f", v))[0]
    return struct.unpack("<Q", struct.pack("<d", v))[0]


def minmax_fp_bits(xs, op: str, width: int) -> int:
    vals = [float(v) for v in xs]
    if any(math.isnan(v) for v in vals):
        return CANONICAL_NAN32 if width == 32 else CANONICAL_NAN64
    if not vals:
        return _bits(math.inf if op == "min" else -math.inf, width)
    pick = min(vals, key=_rank) if op == "min" else max(vals, key=_rank)
    return _bits(pick, width)


def histogram(xs, lo, hi, nbins):
    """Exact-rational histogram: b = floor((x - lo) * nbins / (hi - lo)) with
    Fractions (no rounding at all).  Equal to oracle.c's integer rule for int32;
    for fp32 it differs only where an fp32 rounding moves x across a bin edge
    (none when nbins and hi - lo are powers of two)."""
    from fractions import Fraction
    counts = [0] * nbins
    flo, fhi = Fraction(lo), Fraction(hi)
    for v in xs:
        v = float(v)
        if v != v or not (lo <= v < hi):
            continue
        b = int((Fraction(v) - flo) * nbins / (fhi - flo))
        if 0 <= b < nbins:
            counts[b] += 1
    return counts
