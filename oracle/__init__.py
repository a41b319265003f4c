"""CPU oracle for the device-wide reduction — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import, call, link or execute anything under
``oracle/``.  The product package ``paper_conf_cgo_gonzalohghmh19_b200`` never
imports it, and this package imports nothing from the product: the two share no
code, header, helper, table or constant generator.  Only the seeded input
generators in ``synth/`` (no reduction arithmetic) serve both sides.

What it computes is the plain definition of a reduction — the paper's
sequential atomic-autonomous codelet, Fig. 1(a) (§II.B.1):
``r = x0 (+) x1 (+) ... (+) x_{n-1}`` with ``(+)`` one of the paper's atomic Map
ops add / min / max (§III.A).  The C file ``oracle.c`` holds the
arithmetic; this module compiles it (gcc, ``-O2 -fno-fast-math
-ffp-contract=off``) and wraps it with ctypes.  ``ref.py`` is an independent
exact Python version used to pin ``oracle.c``; ``paper_codelets.py`` replays
the paper's worked examples (Figs. 1–3) step by step.

Every function here is pinned by ``tests/test_oracle.py`` (closed forms,
brute force, permutations, the paper's worked example, special values).
Parity status: all functions pinned (no "parity unpinned" entries).
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

DTYPES = ("int32", "float32", "float64")
OPS = ("sum", "min", "max")

CANONICAL_NAN32 = 0x7FC00000
CANONICAL_NAN64 = 0x7FF8000000000000


def build(force: bool = False) -> str:
    """Compile oracle.c into oracle/liboracle.so (plain gcc, no CUDA)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp",
               "-fPIC", "-shared", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def lib() -> ctypes.CDLL:
    global _lib
    with _lock:
        if _lib is None:
            path = build()
            L = ctypes.CDLL(path)
            vp, sz = ctypes.c_void_p, ctypes.c_size_t
            dp = ctypes.POINTER(ctypes.c_double)
            for name, res, args in [
                ("oracle_sum_i32", ctypes.c_int32, [vp, sz]),
                ("oracle_min_i32", ctypes.c_int32, [vp, sz]),
                ("oracle_max_i32", ctypes.c_int32, [vp, sz]),
                ("oracle_sum_f32", ctypes.c_double, [vp, sz, dp]),
                ("oracle_sum_f64", ctypes.c_double, [vp, sz, dp]),
                ("oracle_min_f32_bits", ctypes.c_uint32, [vp, sz]),
                ("oracle_max_f32_bits", ctypes.c_uint32, [vp, sz]),
                ("oracle_min_f64_bits", ctypes.c_uint64, [vp, sz]),
                ("oracle_max_f64_bits", ctypes.c_uint64, [vp, sz]),
                ("oracle_omp_sum_f32", ctypes.c_float, [vp, sz]),
                ("oracle_omp_threads", ctypes.c_int, []),
                ("oracle_histogram_i32", None, [vp, sz, ctypes.c_double, ctypes.c_double, ctypes.c_int, vp]),
                ("oracle_histogram_f32", None, [vp, sz, ctypes.c_double, ctypes.c_double, ctypes.c_int, vp]),
            ]:
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


class Result:
    """Oracle result.

    ``value``: the exact result for int32 and fp min/max (a numpy scalar of the
    input dtype), or the compensated double sum ``S`` for fp sums.
    ``bits``: the bit pattern the GPU must reproduce exactly (int32 and min/max),
    else None.  ``abs_sum``: ``A = sum |x_i|`` (fp sums only) for the gates.
    """

    __slots__ = ("value", "bits", "abs_sum")

    def __init__(self, value, bits=None, abs_sum=None):
        self.value = value
        self.bits = bits
        self.abs_sum = abs_sum

    def __repr__(self):
        return f"Result(value={self.value!r}, bits={self.bits!r}, abs_sum={self.abs_sum!r})"


def reduce(x: np.ndarray, op: str) -> Result:
    """Reduce a contiguous 1-D numpy array with ``op`` in {'sum','min','max'}."""
    x = np.ascontiguousarray(x)
    if x.ndim != 1:
        x = x.reshape(-1)
    n = x.size
    p = ctypes.c_void_p(x.ctypes.data if n else 0)
    L = lib()
    dt = x.dtype
    if dt == np.int32:
        f = {"sum": L.oracle_sum_i32, "min": L.oracle_min_i32, "max": L.oracle_max_i32}[op]
        v = np.int32(f(p, n))
        return Result(v, bits=int(np.uint32(v.view(np.uint32))))
    if dt == np.float32 or dt == np.float64:
        if op == "sum":
            a = ctypes.c_double(0.0)
            f = L.oracle_sum_f32 if dt == np.float32 else L.oracle_sum_f64
            s = f(p, n, ctypes.byref(a))
            return Result(float(s), abs_sum=float(a.value))
        if dt == np.float32:
            f = L.oracle_min_f32_bits if op == "min" else L.oracle_max_f32_bits
            b = int(f(p, n))
            return Result(np.uint32(b).view(np.float32), bits=b)
        f = L.oracle_min_f64_bits if op == "min" else L.oracle_max_f64_bits
        b = int(f(p, n))
        return Result(np.uint64(b).view(np.float64), bits=b)
    raise TypeError(f"oracle: unsupported dtype {dt}")


def histogram(x: np.ndarray, lo: float, hi: float, nbins: int) -> np.ndarray:
    """Histogram counts (oracle.c, reading R13): exact integer bins for int32,
    fp32 bins floor(fl32(fl32(x - lo) * scale)) for fp32."""
    x = np.ascontiguousarray(x)
    counts = np.zeros(nbins, np.uint32)
    f = lib().oracle_histogram_i32 if x.dtype == np.int32 else lib().oracle_histogram_f32
    if x.dtype not in (np.int32, np.float32):
        raise TypeError("histogram: int32 or float32 input")
    f(ctypes.c_void_p(x.ctypes.data if x.size else 0), x.size, float(lo), float(hi), int(nbins),
      ctypes.c_void_p(counts.ctypes.data))
    return counts


def omp_sum_f32(x: np.ndarray) -> float:
    """The paper-style OpenMP `reduce` pragma baseline; context only."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    return float(lib().oracle_omp_sum_f32(ctypes.c_void_p(x.ctypes.data), x.size))


def omp_threads() -> int:
    return int(lib().oracle_omp_threads())


# ----------------------------------------------------------------- gates ---

EPS = {np.dtype(np.float32): 2.0 ** -23, np.dtype(np.float64): 2.0 ** -52}


def oracle_error_bound(res: Result, dtype, n: int) -> float:
    """Error of the oracle's own S (Neumaier in double): <= 2 u_d |S| + n u_d^2 A."""
    ud = 2.0 ** -53
    return 2 * ud * abs(res.value) + n * ud * ud * res.abs_sum + 1e-300


def gate_g1(res: Result, dtype, n: int) -> float:
    """G1 (north star): |r - S| <= 2 n eps A   (rel <= 2 n eps sum|x| / |sum x|
    multiplied through by |S| so it stays defined at S = 0)."""
    return 2.0 * n * EPS[np.dtype(dtype)] * res.abs_sum + oracle_error_bound(res, dtype, n)


def gate_g2(res: Result, dtype, n: int, chain: int) -> float:
    """G2 (tight): |r - S| <= (L + 1) u A with L the longest addition chain of
    the variant that ran (Higham's gamma_L bound for any summation tree)."""
    u = EPS[np.dtype(dtype)] / 2.0
    return (chain + 1) * u * res.abs_sum + oracle_error_bound(res, dtype, n)


def check_sum(r: float, res: Result, dtype, n: int, chain: int | None = None) -> tuple[bool, str]:
    """Compare a GPU fp sum r against the oracle (non-finite rules R2, gates)."""
    S = res.value
    if math.isnan(S):
        return math.isnan(r), f"expected NaN, got {r!r}"
    if math.isinf(S):
        return r == S, f"expected {S!r}, got {r!r}"
    if not math.isfinite(r):
        return False, f"expected finite {S!r}, got {r!r}"
    err = abs(float(r) - S)
    g1 = gate_g1(res, dtype, n)
    if err > g1:
        return False, f"G1 fail: |r-S|={err:.3e} > {g1:.3e} (r={r!r}, S={S!r})"
    if chain is not None:
        g2 = gate_g2(res, dtype, n, chain)
        if err > g2:
            return False, f"G2 fail: |r-S|={err:.3e} > {g2:.3e} (L={chain}, r={r!r}, S={S!r})"
    return True, f"ok err={err:.3e}"
