/*
 * oracle.c -- plain, slow, obviously-correct CPU reference for the device-wide
 * reduction the paper synthesises GPU code for.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load, call, link or
 * execute anything under oracle/.  The product library
 * (paper_conf_cgo_gonzalohghmh19_b200/) never includes, links or calls this
 * file, and this file includes nothing from the product: it shares no header,
 * helper, constant or table with the CUDA path.
 *
 * What it computes (the plain definition the method reaches, up to fp
 * association):
 *   r = x[0] (+) x[1] (+) ... (+) x[n-1],  (+) in {+, min, max},
 *   r = identity of (+) when n == 0,
 * written as the paper's sequential atomic-autonomous codelet, Fig. 1(a)
 * (section II.B.1): `int accum = 0; for (i ...) accum += in[i];`
 * The op set {add, max, min} is the paper's atomic Map API (section
 * III.A); `atomicSub` is not a reduction (not associative) and is excluded.
 * The element types are the north star's int32 / fp32 / fp64 (the paper's own
 * workload is fp32).
 *
 * Readings of points the paper leaves open (DESIGN.md section "Readings"):
 *   R1 int32 sum wraps modulo 2^32 (two's complement); the paper's `int accum`
 *       never discusses overflow.  Computed in uint32_t.
 *   R2 fp sum: the oracle value S is a compensated (Neumaier) sum carried in
 *      double, plus A = sum |x_i| for the error gates.  Non-finite inputs:
 *      any NaN -> NaN; +inf and -inf both present -> NaN; else any inf -> inf.
 *   R3 fp min/max: NaN anywhere -> canonical quiet NaN (0x7FC00000 /
 *      0x7FF8000000000000); otherwise exact selection with -0.0 < +0.0.
 *   R4 n == 0 -> identity: 0; INT32_MAX / +inf for min; INT32_MIN / -inf for max.
 *
 * Build: gcc -O2 -fno-fast-math -ffp-contract=off -fPIC -shared (oracle/__init__.py).
 */
#include <stddef.h>
#include <stdint.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---------------------------------------------------------------- int32 --- */

/* R1: modular sum, Fig. 1(a) loop with a uint32_t accumulator. */
int32_t oracle_sum_i32(const int32_t* x, size_t n) {
  uint32_t accum = 0u;
  for (size_t i = 0; i < n; ++i) accum += (uint32_t)x[i];
  return (int32_t)accum;
}

int32_t oracle_min_i32(const int32_t* x, size_t n) {
  int32_t m = INT32_MAX;
  for (size_t i = 0; i < n; ++i)
    if (x[i] < m) m = x[i];
  return m;
}

int32_t oracle_max_i32(const int32_t* x, size_t n) {
  int32_t m = INT32_MIN;
  for (size_t i = 0; i < n; ++i)
    if (x[i] > m) m = x[i];
  return m;
}

/* ------------------------------------------------------------ fp sum ----- */

/* Neumaier's improved Kahan summation in double (R2).  `get(i)` is inlined by
 * the two wrappers below.  Returns the non-finite result directly when the
 * input holds NaN or inf (Neumaier itself would turn inf into NaN). */
#define NEUMAIER_BODY(X)                                                      \
  do {                                                                        \
    int has_nan = 0, has_pinf = 0, has_ninf = 0;                              \
    double s = 0.0, c = 0.0, a = 0.0;                                         \
    for (size_t i = 0; i < n; ++i) {                                          \
      double xi = (double)(X)[i];                                             \
      if (isnan(xi)) { has_nan = 1; continue; }                               \
      if (isinf(xi)) { if (xi > 0) has_pinf = 1; else has_ninf = 1; continue; } \
      double t = s + xi;                                                      \
      if (fabs(s) >= fabs(xi)) c += (s - t) + xi;                             \
      else c += (xi - t) + s;                                                 \
      s = t;                                                                  \
      a += fabs(xi);                                                          \
    }                                                                         \
    if (abs_sum) *abs_sum = a;                                                \
    if (has_nan || (has_pinf && has_ninf)) return (double)NAN;               \
    if (has_pinf) return (double)INFINITY;                                    \
    if (has_ninf) return -(double)INFINITY;                                   \
    return s + c;                                                             \
  } while (0)

double oracle_sum_f32(const float* x, size_t n, double* abs_sum) { NEUMAIER_BODY(x); }
double oracle_sum_f64(const double* x, size_t n, double* abs_sum) { NEUMAIER_BODY(x); }

/* ------------------------------------------------------- fp min / max ---- */

/* "a is below b" in the total order used by R3 for non-NaN values:
 * ordinary < , with -0.0 ranked below +0.0 by an explicit sign test. */
static int below_d(double a, double b) {
  if (a < b) return 1;
  if (a == b && a == 0.0 && signbit(a) && !signbit(b)) return 1;
  return 0;
}

uint32_t oracle_min_f32_bits(const float* x, size_t n) {
  float m = INFINITY;
  for (size_t i = 0; i < n; ++i) {
    if (isnan(x[i])) return 0x7FC00000u;
    if (below_d((double)x[i], (double)m)) m = x[i];
  }
  uint32_t b; memcpy(&b, &m, 4); return b;
}

uint32_t oracle_max_f32_bits(const float* x, size_t n) {
  float m = -INFINITY;
  for (size_t i = 0; i < n; ++i) {
    if (isnan(x[i])) return 0x7FC00000u;
    if (below_d((double)m, (double)x[i])) m = x[i];
  }
  uint32_t b; memcpy(&b, &m, 4); return b;
}

uint64_t oracle_min_f64_bits(const double* x, size_t n) {
  double m = INFINITY;
  for (size_t i = 0; i < n; ++i) {
    if (isnan(x[i])) return 0x7FF8000000000000ull;
    if (below_d(x[i], m)) m = x[i];
  }
  uint64_t b; memcpy(&b, &m, 8); return b;
}

uint64_t oracle_max_f64_bits(const double* x, size_t n) {
  double m = -INFINITY;
  for (size_t i = 0; i < n; ++i) {
    if (isnan(x[i])) return 0x7FF8000000000000ull;
    if (below_d(m, x[i])) m = x[i];
  }
  uint64_t b; memcpy(&b, &m, 8); return b;
}

/* ------------------------------------------------------------ histogram --- */

/* the paper motivates shared-memory atomics with histograms
 * (P:L59).  Plain definition (reading R13), bins decided
 * in the input's own arithmetic -- the CUDA side takes the same decisions:
 *   int32: lo, hi integers; x counted iff lo <= x < hi, in bin
 *          b = floor((x - lo) * nbins / (hi - lo))   (exact integer arithmetic);
 *   fp32 : lo_f = (float)lo, hi_f = (float)hi, scale = (float)(nbins / (hi - lo))
 *          (the quotient in double, then rounded to float); x counted iff
 *          lo_f <= x < hi_f and 0 <= b < nbins with
 *          b = floor(fl32(fl32(x - lo_f) * scale))   (two fp32 RN operations).
 * NaN is never counted.  counts is overwritten.
 * The fp32 rule is a definition chosen for the kernel (the paper defines no
 * bin rule); tests/test_oracle.py pins it element by element against the
 * exact-rational bins of oracle/ref.py: they differ only within the rule's
 * rounding reach of a bin edge. */
void oracle_histogram_i32(const int32_t* x, size_t n, double lo, double hi, int nbins, uint32_t* counts) {
  for (int b = 0; b < nbins; ++b) counts[b] = 0u;
  const long long l = (long long)lo, h = (long long)hi;
  const unsigned long long range = (unsigned long long)(h - l);
  for (size_t i = 0; i < n; ++i) {
    const long long v = (long long)x[i];
    if (v < l || v >= h) continue;
    const unsigned long long num = (unsigned long long)(v - l) * (unsigned long long)nbins;
    counts[num / range] += 1u;
  }
}

void oracle_histogram_f32(const float* x, size_t n, double lo, double hi, int nbins, uint32_t* counts) {
  for (int b = 0; b < nbins; ++b) counts[b] = 0u;
  const float lo_f = (float)lo, hi_f = (float)hi;
  const float scale = (float)((double)nbins / (hi - lo));
  for (size_t i = 0; i < n; ++i) {
    const float v = x[i];
    if (!(v >= lo_f && v < hi_f)) continue;
    volatile float d = v - lo_f;   /* each operation rounded to fp32, no contraction */
    volatile float t = d * scale;
    const long long b = (long long)floorf(t);
    if (b >= 0 && b < nbins) counts[b] += 1u;
  }
}

/* --------------------------------------------- paper-style CPU baseline -- */

/* The paper's CPU comparison is an OpenMP 4.0 `reduce` pragma over fp32
 * (P:L469).  This is that loop with a plain float accumulator; it is
 * timed by bench.py as context only, never used to check results. */
float oracle_omp_sum_f32(const float* x, size_t n) {
  float acc = 0.0f;
#pragma omp parallel for reduction(+ : acc) schedule(static)
  for (long long i = 0; i < (long long)n; ++i) acc += x[i];
  return acc;
}

int oracle_omp_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
