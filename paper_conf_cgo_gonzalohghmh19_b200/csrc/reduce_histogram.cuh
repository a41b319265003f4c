// reduce_histogram.cuh -- SURVEY 8(f) N4: a histogram, the workload the paper
// uses to motivate atomics on shared memory, built from
// the same streaming partition as the reduction plus the paper's "VA1"
// codelet (every thread updates a shared accumulator atomically, Fig. 3(a),
// P:L313) with one accumulator per bin.
//
//   counts[b] = #{ i : lo <= x_i < hi, b = floor((x_i - lo) * nbins / (hi - lo)) }
//
// Bins are decided in the input's own arithmetic -- the same rule as the oracle
// (reading R13): int32 exactly -- when (hi - lo) * nbins < 2^32 a
// 32-bit range check and numerator divided by the Granlund-Montgomery
// multiply-high sequence (exact, no correction), else a 64-bit numerator
// divided by multiply-high plus a correction step (no integer division
// instruction either way); fp32 with two correctly rounded fp32
// operations, floor(fl(fl(x - lo) * scale)) (__fsub_rn / __fmul_rn: never
// contracted into an FMA).  The B200's FP64 pipe is far too slow for a
// per-element fp64 rule at HBM speed (measured 2.5 TB/s).  A persistent grid (one wave) streams 32-byte
// vectors (two loads in flight per thread); each block counts into a shared
// histogram (ATOMS.ADD) replicated R times across the banks -- lane l counts
// into copy l % R, so with R = 32 a warp's 32 updates hit 32 different banks
// whatever their bins -- and merges its non-zero bins into `counts` with global
// atomics at the end.  Up to 8 x 16384 bins are split into bin ranges, one range
// per group of blocks (each group re-reads the input); beyond that, elements
// count straight into global memory.
#pragma once
#include "reduce_kernels.cuh"

namespace rb {

constexpr int kHistSharedMaxBins = 16384;  // 64 KB of u32 counters per block
// A/B hooks (profiles/r02_hist_ab.txt, B200, 1 GiB): four vectors in flight
// per thread on the replicated 32-bit path (+2-4 %), the next pair of vectors
// loaded while the 16-bit path updates the current one (+1.6-3.4 %).
#ifndef RB_HIST_V4
#define RB_HIST_V4 1
#endif
#ifndef RB_HIST16_PIPE
#define RB_HIST16_PIPE 1
#endif
// 16-bit path: non-returning shared atomics with block-synchronous flushes
// (k_histogram16r, 65536 bins 3.21 -> 3.78 TB/s fp32, 3.34 -> 3.67 TB/s int32)
// instead of a returning atomic and a carry check per update (k_histogram16);
// RB_HIST16_VPI_{F32,I32} vectors per thread per flush, with the next
// iteration's loads rolled across the flush (RB_HIST16_ROLL; 65536 bins fp32
// 276.6 -> 253.6 us, int32 at 5 vectors 292.9 -> 274.0 us,
// profiles/r02_hist_roll_ab.txt)
#ifndef RB_HIST16_RED
#define RB_HIST16_RED 1
#endif
#ifndef RB_HIST16_ONE_BARRIER
#define RB_HIST16_ONE_BARRIER 1
#endif
#ifndef RB_HIST16_ROLL
#define RB_HIST16_ROLL 1
#endif
#ifndef RB_HIST16_VPI_F32
#define RB_HIST16_VPI_F32 6
#endif
#ifndef RB_HIST16_VPI_I32
#define RB_HIST16_VPI_I32 5
#endif

// Bin of one element, or -1 if it is not counted.  Branch-free (selects and
// predicated corrections), so the bins of a whole vector are computed with
// instruction-level parallelism before any counter is touched.
template <int DT>
__device__ __forceinline__ int hist_bin(uint32_t w, const HistParams& p) {
  if constexpr (DT == DT_I32) {
    if (p.narrow) {  // (hi - lo) * nbins < 2^32: range check and quotient in 32-bit arithmetic
      // int32 range check against the clamped bounds: one subtract, one unsigned compare
      const bool in = w - p.lo_c32 <= p.lim32;
      const unsigned num = (w - p.lo32) * (unsigned)p.nbins;  // x - lo is exact mod 2^32 when counted
      const unsigned t = __umulhi(num, p.magic32);            // exact floor(num / range): no correction
      const unsigned q = (t + ((num - t) >> 1)) >> p.shift32;
      return in ? (int)q : -1;
    }
    const long long v = (long long)(int32_t)w;
    const bool in = v >= p.lo_i && v < p.hi_i;
    int b;
    {
      const unsigned long long num = (unsigned long long)(v - p.lo_i) * (unsigned long long)p.nbins;
      unsigned long long q = __umul64hi(num, p.magic);
      unsigned long long r = num - q * p.range_i;
      if (r >= p.range_i) { ++q; r -= p.range_i; }
      if (r >= p.range_i) ++q;
      b = (int)q;
    }
    return in ? b : -1;
  } else {
    const float x = __uint_as_float(w);
    // x >= lo makes t >= 0, so truncation is floor; t <= nbins * (1 + 2^-22) < 2^31
    const float t = __fmul_rn(__fsub_rn(x, p.lo_f), p.scale_f);
    const int b = __float2int_rz(t);
    return (x >= p.lo_f && x < p.hi_f && b < p.nbins) ? b : -1;  // NaN fails the compares
  }
}

// The same rule in fewer instructions for the shared-memory kernels (nbins <=
// 2^22): the bin as an unsigned value, >= nbins when the element is not
// counted.  fp32: floor(t) for t = fl(fl(x - lo) * scale) in [0, 2^23) is the
// bit pattern of fl_rz(t + 2^23) minus that of 2^23 (the round-toward-zero
// add lands on the integer grid), so no float-to-int conversion; t < 0
// (x < lo) wraps to a huge value, NaN and x >= hi are forced out by the one
// compare left.  The kernels were issue-bound on this arithmetic (ncu,
// profiles/r02_ncu_hist_pairs_vs_16r.json).
#ifndef RB_HIST_UBIN
#define RB_HIST_UBIN 1
#endif
template <int DT>
__device__ __forceinline__ unsigned hist_ubin(uint32_t w, const HistParams& p) {
  if constexpr (DT == DT_I32) {
    if (p.narrow) {
      const bool in = w - p.lo_c32 <= p.lim32;
      const unsigned num = (w - p.lo32) * (unsigned)p.nbins;
      const unsigned t = __umulhi(num, p.magic32);
      const unsigned q = (t + ((num - t) >> 1)) >> p.shift32;
      return in ? q : 0xFFFFFFFFu;
    }
    const int b = hist_bin<DT>(w, p);
    return b < 0 ? 0xFFFFFFFFu : (unsigned)b;
  } else {
#if RB_HIST_UBIN
    const float x = __uint_as_float(w);
    const float t = __fmul_rn(__fsub_rn(x, p.lo_f), p.scale_f);
    const unsigned u = __float_as_uint(__fadd_rz(t, 8388608.0f)) - 0x4B000000u;
    return x < p.hi_f ? u : 0xFFFFFFFFu;
#else
    const int b = hist_bin<DT>(w, p);
    return b < 0 ? 0xFFFFFFFFu : (unsigned)b;
#endif
  }
}

// Count the 8 elements of one vector: bins [b0, b1) in shared memory at byte
// address sbase (this lane's copy; a bin's R copies are adjacent words), or
// straight into global `counts`.
template <int DT, bool kShared>
__device__ __forceinline__ void hist_vec(const uint32_t (&r)[8], const HistParams& p, uint32_t sbase,
                                         uint32_t sdummy, int rshift, int b0, int b1) {
  if constexpr (kShared) {
    unsigned ub[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) ub[k] = hist_ubin<DT>(r[k], p) - (unsigned)b0;  // >= b1 - b0: not counted here
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      // unconditional: an element that is not counted adds to this lane's own
      // dummy word, never merged (ptxas turns any predicated shared atomic
      // into a branch-wrapped one -- a reconvergence region per element)
      const uint32_t a = ub[k] < (unsigned)(b1 - b0) ? sbase + (ub[k] << (rshift + 2)) : sdummy;
      asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(a) : "memory");
    }
  } else {
    int bin[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) bin[k] = hist_bin<DT>(r[k], p);
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (bin[k] >= 0) atomicAdd(p.counts + bin[k], 1u);
  }
}

// kShared: the grid is split into `parts` groups of blocks; group j counts only
// bins [j*K, (j+1)*K) (K = kHistSharedMaxBins) in shared memory, R = 2^rep_log2
// copies per bin, reading the whole input -- `parts` passes over the data
// instead of one global atomic per element.  !kShared: every element is one
// global atomic (very many bins).
#ifndef RB_HIST_MINB_I32
#define RB_HIST_MINB_I32 4  // int32 shared bins at 64 registers: 4 blocks per SM (256 bins 198.7 -> 173.3 us, profiles/r02_hist_i32_minb_ab.txt)
#endif
template <int DT, bool kShared>
__global__ void __launch_bounds__(256, (DT == DT_I32 && kShared) ? RB_HIST_MINB_I32 : 1)
    k_histogram(const HistParams p, int parts, int rep_log2) {
  extern __shared__ unsigned sbins[];
  int b0 = 0, b1 = p.nbins;
  unsigned blk = blockIdx.x, nblk = gridDim.x;
  uint32_t sbase = 0, sdummy = 0;
  if constexpr (kShared) {
    const unsigned per = gridDim.x / parts;
    const unsigned j = blockIdx.x / per;
    blk = blockIdx.x - j * per;
    nblk = per;
    b0 = (int)j * kHistSharedMaxBins;
    b1 = b0 + kHistSharedMaxBins < p.nbins ? b0 + kHistSharedMaxBins : p.nbins;
    const int R = 1 << rep_log2;
    sbase = (uint32_t)__cvta_generic_to_shared(sbins) + 4u * (threadIdx.x & (R - 1));
    // 32 dummy words after the bins, one per lane
    sdummy = (uint32_t)__cvta_generic_to_shared(sbins) + 4u * ((b1 - b0) * R + (threadIdx.x & 31));
    for (int i = threadIdx.x; i < (b1 - b0) * R; i += blockDim.x) sbins[i] = 0u;
    __syncthreads();
  }
  const unsigned long long stride = (unsigned long long)nblk * blockDim.x;
  unsigned long long v = (unsigned long long)blk * blockDim.x + threadIdx.x;
#if RB_HIST_V4
  for (; v + 3 * stride < p.body_vecs; v += 4 * stride) {
    uint32_t r0[8], r1[8], r2[8], r3[8];
    ld_v8(p.body + v * kVecBytes, r0);
    ld_v8(p.body + (v + stride) * kVecBytes, r1);
    ld_v8(p.body + (v + 2 * stride) * kVecBytes, r2);
    ld_v8(p.body + (v + 3 * stride) * kVecBytes, r3);
    hist_vec<DT, kShared>(r0, p, sbase, sdummy, rep_log2, b0, b1);
    hist_vec<DT, kShared>(r1, p, sbase, sdummy, rep_log2, b0, b1);
    hist_vec<DT, kShared>(r2, p, sbase, sdummy, rep_log2, b0, b1);
    hist_vec<DT, kShared>(r3, p, sbase, sdummy, rep_log2, b0, b1);
  }
#endif
  for (; v + stride < p.body_vecs; v += 2 * stride) {
    uint32_t r0[8], r1[8];
    ld_v8(p.body + v * kVecBytes, r0);
    ld_v8(p.body + (v + stride) * kVecBytes, r1);
    hist_vec<DT, kShared>(r0, p, sbase, sdummy, rep_log2, b0, b1);
    hist_vec<DT, kShared>(r1, p, sbase, sdummy, rep_log2, b0, b1);
  }
  if (v < p.body_vecs) {
    uint32_t r[8];
    ld_v8(p.body + v * kVecBytes, r);
    hist_vec<DT, kShared>(r, p, sbase, sdummy, rep_log2, b0, b1);
  }
  if (blk == 0) {  // head and tail elements (< 8 each), as one padded vector
    const int t = threadIdx.x;
    uint32_t r[8];
    const bool mine = t < p.head || (t >= 8 && t - 8 < p.tail);
    r[0] = !mine ? 0u
           : t < p.head ? __ldg((const uint32_t*)p.in + t)
                        : __ldg((const uint32_t*)(p.body + p.body_vecs * kVecBytes) + (t - 8));
    if (mine) {
      const int bn = hist_bin<DT>(r[0], p);
      if constexpr (kShared) {
        if (bn >= b0 && bn < b1)
          asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(sbase + ((uint32_t)(bn - b0) << (rep_log2 + 2))) : "memory");
      } else {
        if (bn >= 0) atomicAdd(p.counts + bn, 1u);
      }
    }
  }
  if constexpr (kShared) {
    __syncthreads();
    // merge: each warp reads 32 consecutive words (32 / R bins, conflict-free),
    // sums each bin's R copies with shuffles, one global atomic per non-zero bin
    const int R = 1 << rep_log2;
    const int lane = threadIdx.x & 31, words = (b1 - b0) * R;
    for (int base = (threadIdx.x & ~31); base < words; base += blockDim.x) {
      const int i = base + lane;
      unsigned c = i < words ? sbins[i] : 0u;
      for (int o = R >> 1; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
      if ((lane & (R - 1)) == 0 && i < words && c) atomicAdd(p.counts + b0 + (i >> rep_log2), c);
    }
  }
}

// Many bins in one pass (16384 < nbins <= ~116 K): one block per SM holds the
// whole histogram as 16-bit counters, two bins per shared word, so 65536 bins
// take 128 KB instead of needing four passes over the input with 32-bit bins.
// A counter is kept below 2^16 by its carry: the update that takes a half from
// 0x7FFF to 0x8000 (seen in the atomic's return value) moves 0x8000 to the
// global count and subtracts it from the half -- exact, and since at most a
// block's in-flight updates (<< 0x8000) can land in between, a half never
// wraps into its neighbour.  The final merge adds both halves of every
// non-zero word to `counts`.
template <int DT>
__global__ void __launch_bounds__(1024) k_histogram16(const HistParams p) {
  extern __shared__ unsigned sw[];
  const int words = (p.nbins + 1) >> 1;
  for (int i = threadIdx.x; i < words + 32; i += blockDim.x) sw[i] = 0u;
  __syncthreads();
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sw);
  const uint32_t sdummy = sbase + 4u * (uint32_t)(words + (threadIdx.x & 31));
  auto count8 = [&](const uint32_t (&r)[8]) {
    int bin[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) bin[k] = hist_bin<DT>(r[k], p);
    uint32_t old[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {  // unconditional (uncounted elements add 0 to the lane's dummy word)
      const bool ok = bin[k] >= 0;
      const uint32_t a = ok ? sbase + 4u * (uint32_t)(bin[k] >> 1) : sdummy;
      const uint32_t inc = ok ? 1u << ((bin[k] & 1) << 4) : 0u;
      asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old[k]) : "r"(a), "r"(inc) : "memory");
    }
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int sh = (bin[k] & 1) << 4;
      if (bin[k] >= 0 && ((old[k] >> sh) & 0xFFFFu) == 0x7FFFu) {  // this update reached 0x8000: carry
        atomicSub(&sw[bin[k] >> 1], 0x8000u << sh);
        atomicAdd(p.counts + bin[k], 0x8000u);
      }
    }
  };
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
#if RB_HIST16_PIPE
  // software pipeline: the next pair of vectors is in flight while this pair's
  // counters are updated (the returning shared atomics of 16 elements take
  // longer than a load round trip under bank conflicts)
  if (v + stride < p.body_vecs) {
    uint32_t r0[8], r1[8];
    ld_v8(p.body + v * kVecBytes, r0);
    ld_v8(p.body + (v + stride) * kVecBytes, r1);
    v += 2 * stride;
    for (; v + stride < p.body_vecs; v += 2 * stride) {
      uint32_t n0[8], n1[8];
      ld_v8(p.body + v * kVecBytes, n0);
      ld_v8(p.body + (v + stride) * kVecBytes, n1);
      count8(r0);
      count8(r1);
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        r0[k] = n0[k];
        r1[k] = n1[k];
      }
    }
    count8(r0);
    count8(r1);
  }
#else
  for (; v + stride < p.body_vecs; v += 2 * stride) {
    uint32_t r0[8], r1[8];
    ld_v8(p.body + v * kVecBytes, r0);
    ld_v8(p.body + (v + stride) * kVecBytes, r1);
    count8(r0);
    count8(r1);
  }
#endif
  if (v < p.body_vecs) {
    uint32_t r[8];
    ld_v8(p.body + v * kVecBytes, r);
    count8(r);
  }
  if (blockIdx.x == 0 && threadIdx.x < 16) {  // head and tail elements (< 8 each)
    const int t = threadIdx.x;
    const bool mine = t < p.head || (t >= 8 && t - 8 < p.tail);
    if (mine) {
      const uint32_t w = t < p.head ? __ldg((const uint32_t*)p.in + t)
                                    : __ldg((const uint32_t*)(p.body + p.body_vecs * kVecBytes) + (t - 8));
      const int bn = hist_bin<DT>(w, p);
      if (bn >= 0) atomicAdd(p.counts + bn, 1u);
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < words; i += blockDim.x) {
    const unsigned w = sw[i];
    if (w & 0xFFFFu) atomicAdd(p.counts + 2 * i, w & 0xFFFFu);
    if (w >> 16) atomicAdd(p.counts + 2 * i + 1, w >> 16);
  }
}

// The same one-pass 16-bit histogram with NON-returning shared atomics
// (red.shared) and block-synchronous flushes instead of a carry check per
// update.  Every iteration each thread counts VPI vectors (8 VPI elements, 8 VPI
// x 1024 per block); then, after a barrier, the block scans its counters and
// moves every half that reached T (the multiple of T it holds) to `counts`.
// After a flush every half is < T and an iteration adds at most 8 VPI x 1024,
// with T + 8 VPI x 1024 <= 0xFFFF: a half never passes 0xFFFF and never
// spills into its neighbour.
// Uniform data never moves anything; the scan costs one 16-byte shared load per
// four words per iteration.
template <int DT>
__global__ void __launch_bounds__(1024) k_histogram16r(const HistParams p) {
  extern __shared__ unsigned sw[];
  const int words = (p.nbins + 1) >> 1;
  const int words4 = (words + 3) & ~3;  // the scan reads uint4
  for (int i = threadIdx.x; i < words4 + 32; i += blockDim.x) sw[i] = 0u;
  __syncthreads();
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sw);
  const uint32_t sdummy = sbase + 4u * (uint32_t)(words4 + (threadIdx.x & 31));
  auto count8 = [&](const uint32_t (&r)[8]) {
    unsigned u[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) u[k] = hist_ubin<DT>(r[k], p);  // >= nbins: not counted
#pragma unroll
    for (int k = 0; k < 8; ++k) {  // unconditional (uncounted elements go to the lane's dummy word, never read)
      const uint32_t a = u[k] < (unsigned)p.nbins ? sbase + 4u * (u[k] >> 1) : sdummy;
      asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a), "r"(1u << ((u[k] & 1u) << 4)) : "memory");
    }
  };
  // VPI vectors per thread per iteration (8 VPI x 1024 elements per block); a
  // half is moved once it reaches T, the largest power of two with
  // T + 8 VPI x 1024 <= 0xFFFF
  constexpr int VPI = DT == DT_I32 ? RB_HIST16_VPI_I32 : RB_HIST16_VPI_F32;
  constexpr unsigned kE = 8u * VPI * 1024u;
  constexpr unsigned kT = kE <= 32767u ? 16384u : (kE <= 49151u ? 16384u >> 1 : (kE <= 57343u ? 4096u : 2048u));
  static_assert(kT + kE <= 0xFFFFu, "a half could wrap");
  constexpr unsigned kHalfMask = (~(kT - 1u)) & 0xFFFFu;
  constexpr unsigned kMask = kHalfMask | (kHalfMask << 16);
  auto flush = [&]() {
#ifdef RB_HIST16_PROBE_NOFLUSH
    return;
#endif
    __syncthreads();
    for (int i = 4 * (int)threadIdx.x; i < words4; i += 4 * (int)blockDim.x) {
      const uint4 w = *reinterpret_cast<const uint4*>(sw + i);
      if (((w.x | w.y | w.z | w.w) & kMask) == 0u) continue;  // every half < T
      const unsigned ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const unsigned lo = ws[j] & kHalfMask, hi = (ws[j] >> 16) & kHalfMask;
        if (lo | hi) {
          atomicSub(&sw[i + j], lo | (hi << 16));
          if (lo) atomicAdd(p.counts + 2 * (i + j), lo);
          if (hi) atomicAdd(p.counts + 2 * (i + j) + 1, hi);
        }
      }
    }
#if !RB_HIST16_ONE_BARRIER
    __syncthreads();
#endif
    // (round 2: no barrier after the scan.  Between two scans of a word only
    // one iteration's updates land -- the first barrier orders every update of
    // iteration i before the scan of flush i, and a thread starts iteration i+1
    // only after its own part of that scan -- and the scan's subtraction only
    // removes what it read, so a half stays < T + E <= 0xFFFF as before.)
  };
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
  // every thread of the block runs the same number of iterations (the barrier
  // in flush): vectors past the body are skipped inside
  const unsigned long long per_iter = VPI * stride;
  const unsigned long long iters = (p.body_vecs + per_iter - 1) / per_iter;
#if RB_HIST16_ROLL
  // rolling loads: vector u of the next iteration is loaded into r[u] as soon
  // as this iteration's vector u is counted, so the next iteration's loads are
  // in flight across the flush and its barriers (1 block per SM: no other
  // block hides the latency there; A/B profiles/r02_hist_roll_ab.txt)
  uint32_t r[VPI][8];
#pragma unroll
  for (int u = 0; u < VPI; ++u)
    if (v + u * stride < p.body_vecs) ld_v8(p.body + (v + u * stride) * kVecBytes, r[u]);
  for (unsigned long long it = 0; it < iters; ++it, v += per_iter) {
    const unsigned long long vn = v + per_iter;
#pragma unroll
    for (int u = 0; u < VPI; ++u) {
      if (v + u * stride < p.body_vecs) count8(r[u]);
      if (vn + u * stride < p.body_vecs) ld_v8(p.body + (vn + u * stride) * kVecBytes, r[u]);
    }
    flush();
  }
#else
  for (unsigned long long it = 0; it < iters; ++it, v += per_iter) {
    uint32_t r[VPI][8];
#pragma unroll
    for (int u = 0; u < VPI; ++u)
      if (v + u * stride < p.body_vecs) ld_v8(p.body + (v + u * stride) * kVecBytes, r[u]);
#pragma unroll
    for (int u = 0; u < VPI; ++u)
      if (v + u * stride < p.body_vecs) count8(r[u]);
    flush();
  }
#endif
  if (blockIdx.x == 0 && threadIdx.x < 16) {  // head and tail elements (< 8 each)
    const int t = threadIdx.x;
    const bool mine = t < p.head || (t >= 8 && t - 8 < p.tail);
    if (mine) {
      const uint32_t w = t < p.head ? __ldg((const uint32_t*)p.in + t)
                                    : __ldg((const uint32_t*)(p.body + p.body_vecs * kVecBytes) + (t - 8));
      const int bn = hist_bin<DT>(w, p);
      if (bn >= 0) atomicAdd(p.counts + bn, 1u);
    }
  }
  __syncthreads();
#ifdef RB_HIST16_PROBE_NOMERGE
  return;
#endif
  // final merge: a word's two halves into counts[2i], counts[2i + 1] with ONE
  // 64-bit global add when both bins exist and no count can carry into its
  // neighbour (p.merge64), else two 32-bit adds -- the 148 x 32768 merge adds
  // are a visible tail at 65 536 bins (fp32 1 GiB: 284 -> 275 us)
  for (int i = threadIdx.x; i < words; i += blockDim.x) {
    const unsigned w = sw[i];
    if (!w) continue;
    if (p.merge64 && 2 * i + 1 < p.nbins) {
      atomicAdd((unsigned long long*)(p.counts + 2 * i), ((unsigned long long)(w >> 16) << 32) | (w & 0xFFFFu));
    } else {
      if (w & 0xFFFFu) atomicAdd(p.counts + 2 * i, w & 0xFFFFu);
      if (w >> 16) atomicAdd(p.counts + 2 * i + 1, w >> 16);
    }
  }
}

#ifndef RB_HIST_REP_MAX
#define RB_HIST_REP_MAX 5
#endif
// Resident blocks per SM of the shared-bin kernel (256 threads each): 4
// (1024 threads) beat the occupancy maximum of 7-8 for fp32 (256 bins 167.9 ->
// 154.0 us; 2 per SM: 181 us; profiles/r02_hist_heur_bps_ab.txt); int32's
// registers allow 3 anyway.
#ifndef RB_HIST_BLOCKS_PER_SM
#define RB_HIST_BLOCKS_PER_SM 4
#endif
// Copies per bin (round 2): only as many as give >= 256 distinct words (few
// bins: one copy per lane group, so a warp's updates do not pile onto a
// handful of addresses); from 256 bins up one copy -- the 32-copy layout
// (lane l -> copy l, conflict-free banks) measured 12-19 % slower there
// (fp32 256 bins 195.0 -> 171.2 us, profiles/r02_hist_rep_bps_ab.txt).
inline int hist_rep_log2(int bins_per_block) {
  int rl = 0;
  while (rl < RB_HIST_REP_MAX && (long long)bins_per_block << rl < 256) ++rl;
  while (rl > 0 && (long long)bins_per_block * (1 << rl) * 4 > 64 * 1024) --rl;
  return rl;
}

template <int DT>
cudaError_t launch_histogram_dt(const HistParams& p, int block, cudaStream_t s) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
#ifdef RB_HIST_PROBE_NOMEMSET
  cudaError_t e = cudaSuccess;  // measurement only: counts are not zeroed
#else
  cudaError_t e = cudaMemsetAsync(p.counts, 0, (size_t)p.nbins * sizeof(unsigned), s);
  if (e != cudaSuccess) return e;
#endif
  if (p.nbins > kHistSharedMaxBins) {  // one pass with 16-bit shared counters if the histogram fits
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    const size_t smem16 = (((size_t)(p.nbins + 1) / 2 + 3) / 4 * 4 + 32) * sizeof(unsigned);
    if (smem16 <= (size_t)optin) {
      auto k16 = RB_HIST16_RED ? k_histogram16r<DT> : k_histogram16<DT>;
      e = opt_in_smem((const void*)k16, (int)smem16);
      if (e != cudaSuccess) return e;
      const int per_sm = blocks_per_sm((const void*)k16, 1024, smem16);
      long long grid = (long long)sms * per_sm;
      const long long need = (long long)((p.body_vecs + 1023) / 1024);
      if (need < grid) grid = need < 1 ? 1 : need;
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3((unsigned)grid, 1, 1);
      cfg.blockDim = dim3(1024, 1, 1);
      cfg.dynamicSmemBytes = smem16;
      cfg.stream = s;
      cfg.numAttrs = 0;
      return cudaLaunchKernelEx(&cfg, k16, p);
    }
  }
  const int parts = (p.nbins + kHistSharedMaxBins - 1) / kHistSharedMaxBins;
  const bool shared = parts <= 8;  // up to 8 passes over the data beat one global atomic per element
  const int per_block_bins = shared ? (parts == 1 ? p.nbins : kHistSharedMaxBins) : 0;
  const int rep_log2 = shared ? hist_rep_log2(per_block_bins) : 0;
  const size_t smem = shared ? ((size_t)per_block_bins * ((size_t)1 << rep_log2) + 32) * sizeof(unsigned) : 0;
  auto kernel = shared ? k_histogram<DT, true> : k_histogram<DT, false>;
  if (smem > 48 * 1024) {
    e = opt_in_smem((const void*)kernel, (int)smem);
    if (e != cudaSuccess) return e;
  }
  // one wave per part group: as many blocks as fit (the shared bins limit residency)
  int per_sm = blocks_per_sm((const void*)kernel, block, smem);
  if (shared && RB_HIST_BLOCKS_PER_SM > 0 && per_sm > RB_HIST_BLOCKS_PER_SM) per_sm = RB_HIST_BLOCKS_PER_SM;
  long long per_part = (long long)sms * per_sm / (shared ? parts : 1);
  const long long need = (long long)((p.body_vecs + block - 1) / block);
  if (need < per_part) per_part = need;
  if (per_part < 1) per_part = 1;
  const long long grid = per_part * (shared ? parts : 1);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.numAttrs = 0;  // follows a memset node: ordinary stream order
  return cudaLaunchKernelEx(&cfg, kernel, p, shared ? parts : 1, rep_log2);
}

}  // namespace rb
