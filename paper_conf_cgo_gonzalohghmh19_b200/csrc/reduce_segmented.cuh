// reduce_segmented.cuh -- many independent reductions in one launch (SURVEY
// section 8(f) N1: batched / segmented reduction).
//
// Segment i is in[lo_i, hi_i) with lo_i = offsets[i], hi_i = offsets[i+1]
// (device int64 array of num_segments + 1 entries), or lo_i = i * seg_len for
// uniform batches (offsets == NULL); out[i] receives its result.  The paper's
// small-array winners assign one warp or one block per
// partition with no global atomics; here the group size is chosen from the mean
// segment length:
//   kGroup == 32    : one warp per segment (8 segments per 256-thread block),
//                     warp combine only (redux / shuffles);
//   kGroup == block : one block per segment, block combine "Vs".
// Each segment gets its own head / 32-byte-aligned body / tail split, so any
// element-aligned offset works.  Every step is fixed-order: deterministic.
#pragma once
#include "reduce_kernels.cuh"

namespace rb {

// Fold in[lo, hi) by `lanes` cooperating threads (this one is `lid`).
template <class T, int U>
__device__ __forceinline__ void fold_range(Part<T> (&a)[T::NA], uint32_t& aux, const char* base,
                                           long long lo, long long hi, int lid, int lanes) {
  using Elem = typename T::Elem;
  constexpr int s = sizeof(Elem);
  if (hi <= lo) return;
  const char* p = base + lo * s;
  const long long n = hi - lo;
  const unsigned mis = (unsigned)((uintptr_t)p & 31u);
  long long head = mis ? (long long)((32u - mis) / s) : 0;
  if (head > n) head = n;
  const char* body = p + head * s;
  const long long nvec = (n - head) / T::VE;
  const long long tail = (n - head) % T::VE;
  long long v = lid;
  for (; v + (long long)(U - 1) * lanes < nvec; v += (long long)U * lanes) {
    uint32_t r[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) ld_v8(body + (v + (long long)u * lanes) * kVecBytes, r[u]);
#pragma unroll
    for (int u = 0; u < U; ++u) fold_vec<T>(a, aux, r[u], u);
  }
  for (; v < nvec; v += lanes) {
    uint32_t r[8];
    ld_v8(body + v * kVecBytes, r);
    fold_vec<T>(a, aux, r, 0);
  }
  // head and tail (< 8 elements each) by the first lanes, into two different
  // accumulators (groups may be only 8 lanes wide)
  if (lid < head) fold_elem<T>(a[0], aux, __ldg((const Elem*)p + lid));
  if (lid < tail) fold_elem<T>(a[T::NA - 1], aux, __ldg((const Elem*)(body + nvec * kVecBytes) + lid));
}

template <class T>
__device__ __forceinline__ void seg_store(const SegParams& p, long long seg, typename T::Grid g) {
  if (p.raw_out) ((typename T::Grid*)p.out)[seg] = g;
  else T::finalize(g, (char*)p.out + seg * (long long)sizeof(typename T::Elem));
}

// kGroup = 8 or 32: that many lanes per segment (4 or 1 segments per warp in
// flight); kGroup = 0: one block per segment.  The grid is persistent (a few
// blocks per SM) and groups stride over the segments, so millions of tiny
// segments do not pay one CTA launch each.
template <int DT, int OP, int kGroup>
__global__ void __launch_bounds__(512) k_segmented(const SegParams p) {
  using T = Tr<DT, OP>;
  using Acc = typename T::Acc;
  pdl_wait();
  const int lane = threadIdx.x & 31;
  long long first, step;
  int lid, lanes;
  if constexpr (kGroup > 0) {
    const long long groups_per_block = blockDim.x / kGroup;
    first = (long long)blockIdx.x * groups_per_block + threadIdx.x / kGroup;
    step = (long long)gridDim.x * groups_per_block;
    lid = threadIdx.x % kGroup;
    lanes = kGroup;
  } else {
    first = blockIdx.x;
    step = gridDim.x;
    lid = threadIdx.x;
    lanes = blockDim.x;
  }
  // all groups of a warp (all threads of a block) run the same number of
  // iterations -- the shuffles / barriers need every lane -- and a group past
  // the last segment folds nothing
  const long long base = kGroup > 0 ? first - lane / kGroup : first;
  const long long iters = base < p.nseg ? (p.nseg - base + step - 1) / step : 0;
#pragma unroll 1
  for (long long it = 0; it < iters; ++it) {
    const long long seg = first + it * step;
    const bool live = seg < p.nseg;
    long long lo = 0, hi = 0;
    if (live) {
      if (p.offsets) {
        lo = __ldg(p.offsets + seg);
        hi = __ldg(p.offsets + seg + 1);
      } else {
        lo = seg * p.seg_len;
        hi = lo + p.seg_len;
      }
    }
    Part<T> a[T::NA];
    init_parts<T>(a);
    uint32_t aux = 0;
    fold_range<T, 4>(a, aux, p.in, lo, hi, lid, lanes);
    const Acc v = thread_result<T>(a, aux);
    if constexpr (kGroup == 32) {
      const Acc w = T::warp(v);
      if (lane == 0 && live) seg_store<T>(p, seg, T::to_grid(w));
    } else if constexpr (kGroup > 0) {
      Acc w = v;
#pragma unroll
      for (int o = kGroup / 2; o > 0; o >>= 1) w = T::comb(w, shfl_xor(w, o));
      if (lid == 0 && live) seg_store<T>(p, seg, T::to_grid(w));
    } else {
      const typename T::Grid g = block_combine<T, BC_SHFL>(v);
      if (threadIdx.x == 0 && live) seg_store<T>(p, seg, g);
      __syncthreads();  // block_combine's shared scratch is reused next iteration
    }
  }
  pdl_trigger();  // persistent grid: let the next kernel in only as this one finishes
}

template <int DT, int OP>
cudaError_t launch_segmented_op(const SegParams& p, int group, int block, cudaStream_t s) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long per_block = group > 0 ? block / group : 1;
  long long grid = (p.nseg + per_block - 1) / per_block;
  const long long cap = (long long)sms * (2048 / block);  // one full wave
  if (grid > cap) grid = cap;
  if (grid < 1) grid = 1;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  if (group == 8) return cudaLaunchKernelEx(&cfg, k_segmented<DT, OP, 8>, p);
  if (group == 32) return cudaLaunchKernelEx(&cfg, k_segmented<DT, OP, 32>, p);
  return cudaLaunchKernelEx(&cfg, k_segmented<DT, OP, 0>, p);
}

template <int DT>
cudaError_t launch_segmented_dt(int op, const SegParams& p, int group, int block, cudaStream_t s) {
  switch (op) {
    case OP_SUM: return launch_segmented_op<DT, OP_SUM>(p, group, block, s);
    case OP_MIN: return launch_segmented_op<DT, OP_MIN>(p, group, block, s);
    case OP_MAX: return launch_segmented_op<DT, OP_MAX>(p, group, block, s);
    case OP_SUMACC:
      if constexpr (DT != DT_I32) return launch_segmented_op<DT, OP_SUMACC>(p, group, block, s);
      break;
  }
  return cudaErrorInvalidValue;
}

}  // namespace rb
