// reduce_histogram.cuh -- SURVEY 8(f) N4: a histogram, the workload the paper
// uses to motivate atomics on shared memory, built from
// the same streaming partition as the reduction plus the paper's "VA1"
// codelet (every thread updates a shared accumulator atomically, Fig. 3(a),
// P:L313) with one accumulator per bin.
//
//   counts[b] = #{ i : lo <= x_i < hi, b = floor((x_i - lo) * nbins / (hi - lo)) }
//
// The bin is decided in fp64 with one subtraction, one multiplication and one
// division, each rounded to nearest and never contracted into an FMA (the
// __d*_rn intrinsics) -- the same rule, in the same precision, as the oracle
// (reading R13).  A persistent grid (one wave) streams 32-byte
// vectors; each block counts into a shared histogram (ATOMS.ADD) and merges
// its non-zero bins into `counts` with global atomics at the end; bin counts
// beyond the shared-memory budget count straight into global memory.
#pragma once
#include "reduce_kernels.cuh"

namespace rb {

constexpr int kHistSharedMaxBins = 16384;  // 64 KB of u32 counters per block

template <bool kShared>
__device__ __forceinline__ void hist_add(double x, const HistParams& p, unsigned* bins) {
  if (!(x >= p.lo && x < p.hi)) return;  // NaN fails both
  double t = __dsub_rn(x, p.lo);
  t = __dmul_rn(t, (double)p.nbins);
  t = __ddiv_rn(t, p.range);
  const long long b = (long long)floor(t);
  if (b >= 0 && b < p.nbins) atomicAdd(bins + b, 1u);
}

template <int DT, bool kShared>
__global__ void __launch_bounds__(512) k_histogram(const HistParams p) {
  extern __shared__ unsigned sbins[];
  unsigned* bins = kShared ? sbins : p.counts;
  if constexpr (kShared) {
    for (int i = threadIdx.x; i < p.nbins; i += blockDim.x) sbins[i] = 0u;
    __syncthreads();
  }
  const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
  unsigned long long v = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
  for (; v < p.body_vecs; v += stride) {
    uint32_t r[8];
    ld_v8(p.body + v * kVecBytes, r);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const double x = DT == DT_I32 ? (double)(int32_t)r[k] : (double)__uint_as_float(r[k]);
      hist_add<kShared>(x, p, bins);
    }
  }
  if (blockIdx.x == 0) {
    const int t = threadIdx.x;
    if (t < p.head) {
      const uint32_t w = __ldg((const uint32_t*)p.in + t);
      hist_add<kShared>(DT == DT_I32 ? (double)(int32_t)w : (double)__uint_as_float(w), p, bins);
    } else if (t >= 8 && t - 8 < p.tail) {
      const uint32_t w = __ldg((const uint32_t*)(p.body + p.body_vecs * kVecBytes) + (t - 8));
      hist_add<kShared>(DT == DT_I32 ? (double)(int32_t)w : (double)__uint_as_float(w), p, bins);
    }
  }
  if constexpr (kShared) {
    __syncthreads();
    for (int i = threadIdx.x; i < p.nbins; i += blockDim.x) {
      const unsigned c = sbins[i];
      if (c) atomicAdd(p.counts + i, c);
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
  const bool shared = p.nbins <= kHistSharedMaxBins;
  const size_t smem = shared ? (size_t)p.nbins * sizeof(unsigned) : 0;
  // one wave: as many blocks as fit (shared histogram size limits residency)
  int per_sm = 2048 / block;
  if (shared && smem > 0) {
    const int by_smem = (int)((200 * 1024) / smem);
    if (by_smem < per_sm) per_sm = by_smem < 1 ? 1 : by_smem;
  }
  long long grid = (long long)sms * per_sm;
  const long long need = (long long)((p.body_vecs + block - 1) / block);
  if (need < grid) grid = need < 1 ? 1 : need;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 0;  // follows a memset node: ordinary stream order
  if (shared) {
    if (smem > 48 * 1024) {
      e = cudaFuncSetAttribute(k_histogram<DT, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               kHistSharedMaxBins * (int)sizeof(unsigned));
      if (e != cudaSuccess) return e;
    }
    return cudaLaunchKernelEx(&cfg, k_histogram<DT, true>, p);
  }
  return cudaLaunchKernelEx(&cfg, k_histogram<DT, false>, p);
}

}  // namespace rb
