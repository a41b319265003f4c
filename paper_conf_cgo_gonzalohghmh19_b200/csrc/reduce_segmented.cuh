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
__device__ __forceinline__ void fold_range(typename T::Acc (&a)[T::NA], uint32_t& aux, const char* base,
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
    for (int u = 0; u < U; ++u) fold_vec<T>(a, aux, r[u]);
  }
  for (; v < nvec; v += lanes) {
    uint32_t r[8];
    ld_v8(body + v * kVecBytes, r);
    fold_vec<T>(a, aux, r);
  }
  if (lid < head) fold_elem<T>(a[0], aux, __ldg((const Elem*)p + lid));
  if (lid >= 8 && lid - 8 < tail) fold_elem<T>(a[0], aux, __ldg((const Elem*)(body + nvec * kVecBytes) + (lid - 8)));
}

template <class T>
__device__ __forceinline__ void seg_store(const SegParams& p, long long seg, typename T::Grid g) {
  if (p.raw_out) ((typename T::Grid*)p.out)[seg] = g;
  else T::finalize(g, (char*)p.out + seg * (long long)sizeof(typename T::Elem));
}

template <int DT, int OP, bool kWarpPerSeg>
__global__ void __launch_bounds__(1024) k_segmented(const SegParams p) {
  using T = Tr<DT, OP>;
  using Acc = typename T::Acc;
  pdl_wait();
  if (blockIdx.x + kPdlTriggerWindow >= gridDim.x) pdl_trigger();
  const int lane = threadIdx.x & 31;
  long long seg;
  int lid, lanes;
  if constexpr (kWarpPerSeg) {
    seg = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    lid = lane;
    lanes = 32;
    if (seg >= p.nseg) return;  // whole warp leaves together
  } else {
    seg = blockIdx.x;
    lid = threadIdx.x;
    lanes = blockDim.x;
  }
  long long lo, hi;
  if (p.offsets) {
    lo = __ldg(p.offsets + seg);
    hi = __ldg(p.offsets + seg + 1);
  } else {
    lo = seg * p.seg_len;
    hi = lo + p.seg_len;
  }
  Acc a[T::NA];
#pragma unroll
  for (int k = 0; k < T::NA; ++k) a[k] = T::ident();
  uint32_t aux = 0;
  fold_range<T, 4>(a, aux, p.in, lo, hi, lid, lanes);
  const Acc v = thread_result<T>(a, aux);
  if constexpr (kWarpPerSeg) {
    const Acc w = T::warp(v);
    if (lane == 0) seg_store<T>(p, seg, T::to_grid(w));
  } else {
    const typename T::Grid g = block_combine<T, BC_SHFL>(v);
    if (threadIdx.x == 0) seg_store<T>(p, seg, g);
  }
}

template <int DT, int OP>
cudaError_t launch_segmented_op(const SegParams& p, bool warp_per_seg, int block, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  const long long per_block = warp_per_seg ? block / 32 : 1;
  const long long grid = (p.nseg + per_block - 1) / per_block;
  if (grid > 0x7FFFFFFFll) return cudaErrorInvalidValue;
  cfg.gridDim = dim3((unsigned)grid, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  if (warp_per_seg) return cudaLaunchKernelEx(&cfg, k_segmented<DT, OP, true>, p);
  return cudaLaunchKernelEx(&cfg, k_segmented<DT, OP, false>, p);
}

template <int DT>
cudaError_t launch_segmented_dt(int op, const SegParams& p, bool warp_per_seg, int block, cudaStream_t s) {
  switch (op) {
    case OP_SUM: return launch_segmented_op<DT, OP_SUM>(p, warp_per_seg, block, s);
    case OP_MIN: return launch_segmented_op<DT, OP_MIN>(p, warp_per_seg, block, s);
    case OP_MAX: return launch_segmented_op<DT, OP_MAX>(p, warp_per_seg, block, s);
  }
  return cudaErrorInvalidValue;
}

}  // namespace rb
