// reduce_histogram.cuh -- SURVEY 8(f) N4: a histogram, the workload the paper
// uses to motivate atomics on shared memory, built from
// the same streaming partition as the reduction plus the paper's "VA1"
// codelet (every thread updates a shared accumulator atomically, Fig. 3(a),
// P:L313) with one accumulator per bin.
//
//   counts[b] = #{ i : lo <= x_i < hi, b = floor((x_i - lo) * nbins / (hi - lo)) }
//
// Bins are decided in the input's own arithmetic -- the same rule as the oracle
// (reading R13): int32 exactly, with a 64-bit numerator divided by
// multiply-high with a precomputed reciprocal plus a correction step (no
// integer division instruction); fp32 with two correctly rounded fp32
// operations, floor(fl(fl(x - lo) * scale)) (__fsub_rn / __fmul_rn: never
// contracted into an FMA).  The B200's FP64 pipe is far too slow for a
// per-element fp64 rule at HBM speed (measured 2.5 TB/s).  A persistent grid (one wave) streams 32-byte
// vectors; each block counts into a shared histogram (ATOMS.ADD) and merges
// its non-zero bins into `counts` with global atomics at the end.  Up to 8 x
// 16384 bins are split into bin ranges, one range per group of blocks (each
// group re-reads the input); beyond that, elements count straight into global
// memory.
#pragma once
#include "reduce_kernels.cuh"

namespace rb {

constexpr int kHistSharedMaxBins = 16384;  // 64 KB of u32 counters per block

// Count w into bins[b - b0] if its bin b lies in [b0, b1).
template <int DT>
__device__ __forceinline__ void hist_add(uint32_t w, const HistParams& p, unsigned* bins, long long b0, long long b1) {
  if constexpr (DT == DT_I32) {
    const long long v = (long long)(int32_t)w;
    if (v < p.lo_i || v >= p.hi_i) return;
    const unsigned long long num = (unsigned long long)(v - p.lo_i) * (unsigned long long)p.nbins;
    unsigned long long q = __umul64hi(num, p.magic);
    unsigned long long r = num - q * p.range_i;
    while (r >= p.range_i) {  // at most two steps: q underestimates by < 2
      ++q;
      r -= p.range_i;
    }
    if ((long long)q >= b0 && (long long)q < b1) atomicAdd(bins + (q - b0), 1u);
  } else {
    const float x = __uint_as_float(w);
    if (!(x >= p.lo_f && x < p.hi_f)) return;  // NaN fails both
    const float t = __fmul_rn(__fsub_rn(x, p.lo_f), p.scale_f);
    const long long b = (long long)floorf(t);
    if (b >= 0 && b < p.nbins && b >= b0 && b < b1) atomicAdd(bins + (b - b0), 1u);
  }
}

// kShared: the grid is split into `parts` groups of blocks; group j counts only
// bins [j*K, (j+1)*K) (K = kHistSharedMaxBins) in shared memory, reading the
// whole input -- `parts` passes over the data instead of one global atomic per
// element.  !kShared: every element is one global atomic (very many bins).
template <int DT, bool kShared>
__global__ void __launch_bounds__(512) k_histogram(const HistParams p, int parts) {
  extern __shared__ unsigned sbins[];
  long long b0 = 0, b1 = p.nbins;
  unsigned blk = blockIdx.x, nblk = gridDim.x;
  unsigned* bins = p.counts;
  if constexpr (kShared) {
    const unsigned per = gridDim.x / parts;
    const unsigned j = blockIdx.x / per;
    blk = blockIdx.x - j * per;
    nblk = per;
    b0 = (long long)j * kHistSharedMaxBins;
    b1 = b0 + kHistSharedMaxBins < p.nbins ? b0 + kHistSharedMaxBins : p.nbins;
    bins = sbins;
    for (long long i = threadIdx.x; i < b1 - b0; i += blockDim.x) sbins[i] = 0u;
    __syncthreads();
  }
  const unsigned long long stride = (unsigned long long)nblk * blockDim.x;
  unsigned long long v = (unsigned long long)blk * blockDim.x + threadIdx.x;
  for (; v < p.body_vecs; v += stride) {
    uint32_t r[8];
    ld_v8(p.body + v * kVecBytes, r);
#pragma unroll
    for (int k = 0; k < 8; ++k) hist_add<DT>(r[k], p, bins, b0, b1);
  }
  if (blk == 0) {
    const int t = threadIdx.x;
    if (t < p.head) hist_add<DT>(__ldg((const uint32_t*)p.in + t), p, bins, b0, b1);
    else if (t >= 8 && t - 8 < p.tail)
      hist_add<DT>(__ldg((const uint32_t*)(p.body + p.body_vecs * kVecBytes) + (t - 8)), p, bins, b0, b1);
  }
  if constexpr (kShared) {
    __syncthreads();
    for (long long i = threadIdx.x; i < b1 - b0; i += blockDim.x) {
      const unsigned c = sbins[i];
      if (c) atomicAdd(p.counts + b0 + i, c);
    }
  }
}

template <int DT>
cudaError_t launch_histogram_dt(const HistParams& p, int block, cudaStream_t s) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaError_t e = cudaMemsetAsync(p.counts, 0, (size_t)p.nbins * sizeof(unsigned), s);
  if (e != cudaSuccess) return e;
  const int parts = (p.nbins + kHistSharedMaxBins - 1) / kHistSharedMaxBins;
  const bool shared = parts <= 8;  // up to 8 passes over the data beat one global atomic per element
  const int sbins = shared ? (parts == 1 ? p.nbins : kHistSharedMaxBins) : 0;
  const size_t smem = (size_t)sbins * sizeof(unsigned);
  // one wave per part group: as many blocks as fit (the shared bins limit residency)
  int per_sm = 2048 / block;
  if (smem > 0) {
    const int by_smem = (int)((200 * 1024) / smem);
    if (by_smem < per_sm) per_sm = by_smem < 1 ? 1 : by_smem;
  }
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
  if (shared) {
    if (smem > 48 * 1024) {
      e = cudaFuncSetAttribute(k_histogram<DT, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               kHistSharedMaxBins * (int)sizeof(unsigned));
      if (e != cudaSuccess) return e;
    }
    return cudaLaunchKernelEx(&cfg, k_histogram<DT, true>, p, parts);
  }
  return cudaLaunchKernelEx(&cfg, k_histogram<DT, false>, p, 1);
}

}  // namespace rb
