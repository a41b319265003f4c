// reduce_segbal.cuh -- element-balanced segmented reduction of an offsets
// array (the variable-length case).
//
// reduce_segmented's group kernels give every segment to one group, so the
// time a group spends depends on the lengths it draws: with power-law lengths
// the grid waits for the few groups that drew long segments, and each short
// segment costs a chain of dependent loads (offsets -> data -> store).  Here
// the ELEMENTS are split evenly instead: the flat range [offsets[0],
// offsets[nseg]) is cut into 8 KB chunks on 32-byte boundaries and one warp
// reduces one chunk whatever the segments inside it look like -- the
// partition is by data, as the paper's tiled distribution of a single array
// (Fig. 1(b)), with segment boundaries carried inside it.
//
//   k_segbal_scan : one thread per segment: the identity for empty segments,
//                   start_seg[c] = the segment holding chunk c's first element,
//                   and a flag if the offsets are not monotone (then the chunk
//                   kernel falls back to one warp per segment).
//   k_segbal      : one warp per chunk.  Lane l owns the chunk's 256 bytes
//                   [256 l, 256 l + 256) (eight 32-byte loads in flight).  The
//                   chunk's slice of the offsets array is copied into shared
//                   memory as chunk-local positions; each lane turns the
//                   boundaries in its range into a 64-bit mask, folds its
//                   elements in order, closing a piece at every set bit
//                   (pieces go to shared memory).  A segmented scan over the
//                   32 lanes (5 shuffle steps, fixed order) joins the pieces of
//                   segments that cross lanes.  Segments that start and end in
//                   the chunk are written directly; the chunk leaves its first
//                   piece (the segment that began before it) and its last piece
//                   (the segment still open at its end) for the fix-up.  A chunk
//                   without boundaries folds with the plain vector tree.
//   k_segbal_fix  : one warp per chunk whose last piece opens a segment: joins
//                   it with the first pieces of the following chunks up to the
//                   chunk where the segment closes (32 chunks per step, fixed
//                   order), writes out[segment], and the last block resets the
//                   call's flags.
// Values never touch atomics and every combine order depends only on the
// offsets: deterministic.  Chunk geometry depends only on the input address
// modulo 32 and offsets[0].
#pragma once
#include "reduce_segmented.cuh"

namespace rb {

constexpr int kBalWarps = 4;        // warps per block of k_segbal
constexpr int kBalVecsPerLane = 8;  // 32-byte vectors per lane per chunk (256 contiguous bytes)

template <class T>
struct Bal {
  using Acc = typename T::Acc;
  static constexpr int s = sizeof(typename T::Elem);
  static constexpr int EL = kBalVecsPerLane * T::VE;  // elements per lane (64 or 32)
  static constexpr long long C = 32LL * EL;           // elements per chunk (8 KB)
  static constexpr int kList = (int)C + 64;           // offsets entries kept in shared memory
  static constexpr size_t kPieceBytes = (size_t)EL * 32 * sizeof(Acc);
  static constexpr size_t kListBytes = ((size_t)kList * 2 + 15) / 16 * 16;
  static constexpr size_t kWarpSmem = kPieceBytes + kListBytes;
};

// Element index (relative to `in`) of the 32-byte-aligned address at or below
// in + E0: chunk c covers [P0 + c*C, P0 + (c+1)*C) clipped to [E0, E1).
template <int S>
__device__ __forceinline__ long long bal_origin(const char* in, long long E0) {
  const unsigned mis = (unsigned)(((uintptr_t)in + (uintptr_t)(E0 * S)) & 31u);
  return E0 - (long long)(mis / S);
}

template <class T>
__device__ __forceinline__ typename T::Elem elem_ident() {
  if constexpr (std::is_same<typename T::Acc, double2>::value) return 0.0;
  else return (typename T::Elem)T::ident();
}

// element e of a lane's 8 vectors (e is a constant after unrolling)
template <class T>
__device__ __forceinline__ typename T::Elem bal_elem(const uint32_t (&r)[kBalVecsPerLane][8], int e) {
  using Elem = typename T::Elem;
  if constexpr (sizeof(Elem) == 4) {
    const uint32_t w = r[e / 8][e % 8];
    return *reinterpret_cast<const Elem*>(&w);
  } else {
    return __hiloint2double((int)r[e / 4][2 * (e % 4) + 1], (int)r[e / 4][2 * (e % 4)]);
  }
}

// one element into a piece: the traits' streaming fold, except fp64 min/max,
// whose streaming fold defers NaN to a per-thread flag -- pieces use the full
// NaN-propagating combine instead (a piece may be closed after any element)
template <class T>
__device__ __forceinline__ void bal_fold1(Part<T>& a, uint32_t& aux, typename T::Elem x) {
  if constexpr (HasSelNaN<T>::value) a = T::comb(a, x);
  else fold_elem<T>(a, aux, x);
}

template <class V>
__device__ __forceinline__ V shfl_up_v(V v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
__device__ __forceinline__ double2 shfl_up_v(double2 v, int d) {
  return make_double2(__shfl_up_sync(0xffffffffu, v.x, d), __shfl_up_sync(0xffffffffu, v.y, d));
}

template <class T>
__device__ __forceinline__ void bal_store(const SegParams& p, long long seg, typename T::Grid g) {
  if (seg < p.nseg) seg_store<T>(p, seg, g);
}

// Warp-cooperative value of in[lo, hi) (result in every lane).
template <class T>
__device__ __forceinline__ typename T::Acc bal_warp_range(const SegParams& p, long long lo, long long hi, int lane) {
  Part<T> a[T::NA];
  init_parts<T>(a);
  uint32_t aux = 0;
  fold_range<T, 4>(a, aux, p.in, lo, hi, lane, 32);
  return T::warp(thread_result<T>(a, aux));
}

template <int DT, int OP>
__global__ void __launch_bounds__(256) k_segbal_scan(const SegParams p) {
  using T = Tr<DT, OP>;
  using B = Bal<T>;
  pdl_wait();
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < p.nseg) {
    const long long E0 = __ldg(p.offsets), lo = __ldg(p.offsets + i), hi = __ldg(p.offsets + i + 1);
    if (hi < lo) atomicOr(p.b.hdr, 1u);
    if (hi <= lo) {
      seg_store<T>(p, i, T::gident());
    } else {
      const long long P0 = bal_origin<B::s>(p.in, E0);
      long long c0 = lo <= E0 ? 0 : (lo - P0 + B::C - 1) / B::C;  // chunks starting in [lo, hi)
      long long c1 = (hi - P0 + B::C - 1) / B::C;
      if (c1 > (long long)kBalChunks) c1 = kBalChunks;
      for (long long c = c0; c < c1; ++c) p.b.start_seg[c] = (unsigned)i;
    }
  }
  pdl_trigger();
}

// The slow path of one chunk (its offsets slice does not fit the shared list:
// thousands of empty segments): walk the segments in global memory, one warp
// fold per piece.  Same outputs as the fast path.
template <class T>
__device__ __forceinline__ void bal_chunk_walk(const SegParams& p, long long c, long long clo, long long chi,
                                            long long E0, long long E1, unsigned s0, int lane) {
  using Grid = typename T::Grid;
  const long long nseg = p.nseg;
  const long long vlo = clo > E0 ? clo : E0, vhi = chi < E1 ? chi : E1;
  long long j = s0;
  bool incoming = __ldg(p.offsets + j) < clo;
  unsigned has_b = incoming ? 0u : 1u;
  Grid first = T::gident(), last = T::gident();
  unsigned lseg = 0xFFFFFFFFu;
  long long pos = vlo;
  while (true) {
    const long long end = __ldg(p.offsets + j + 1);
    const typename T::Acc v = bal_warp_range<T>(p, pos, end < vhi ? end : vhi, lane);
    if (end < chi) {  // segment j closes inside the chunk
      if (incoming) {
        first = T::to_grid(v);
        incoming = false;
        has_b = 1u;
      } else if (lane == 0) {
        bal_store<T>(p, j, T::to_grid(v));
      }
      long long i = j + 1;  // the non-empty segment starting at `end`
      while (i < nseg && __ldg(p.offsets + i + 1) == end) ++i;
      j = i;
      pos = end;
      if (j >= nseg) break;
    } else {
      if (incoming) first = last = T::to_grid(v);
      else { last = T::to_grid(v); lseg = (unsigned)j; }
      break;
    }
  }
  if (lane == 0) {
    ((Grid*)p.b.first_val)[c] = first;
    ((Grid*)p.b.last_val)[c] = last;
    p.b.flags[c] = has_b;
    p.b.last_seg[c] = lseg;
  }
}

template <int DT, int OP>
__global__ void __launch_bounds__(kBalWarps * 32) k_segbal(const SegParams p) {
  using T = Tr<DT, OP>;
  using B = Bal<T>;
  using Acc = typename T::Acc;
  using Elem = typename T::Elem;
  using Grid = typename T::Grid;
  extern __shared__ __align__(16) unsigned char bal_smem[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  Acc* pieces = reinterpret_cast<Acc*>(bal_smem + wib * B::kWarpSmem);
  short* list = reinterpret_cast<short*>(bal_smem + wib * B::kWarpSmem + B::kPieceBytes);
  pdl_wait();
  const long long nseg = p.nseg;
  const long long E0 = __ldg(p.offsets), E1 = __ldg(p.offsets + nseg);
  const unsigned nonmono = *(volatile unsigned*)p.b.hdr;
  const long long P0 = bal_origin<B::s>(p.in, E0);
  const long long nchunks = E1 > E0 ? (E1 - P0 + B::C - 1) / B::C : 0;
  const long long gw = (long long)blockIdx.x * kBalWarps + wib, nw = (long long)gridDim.x * kBalWarps;
  if (nonmono || nchunks > (long long)kBalChunks) {
    // offsets not monotone (overlapping segments) or more chunks than the
    // workspace holds: one warp per segment
#pragma unroll 1
    for (long long seg = gw; seg < nseg; seg += nw) {
      const long long lo = __ldg(p.offsets + seg), hi = __ldg(p.offsets + seg + 1);
      if (hi <= lo) continue;
      const Acc w = bal_warp_range<T>(p, lo, hi, lane);
      if (lane == 0) seg_store<T>(p, seg, T::to_grid(w));
    }
    pdl_trigger();
    return;
  }
  const Elem eid = elem_ident<T>();
#pragma unroll 1
  for (long long c = gw; c < nchunks; c += nw) {
    const long long clo = P0 + c * B::C, chi = clo + B::C;
    const unsigned s0 = __ldcg(p.b.start_seg + c);
    // 1. the lane's 256 bytes, all loads in flight
    uint32_t r[kBalVecsPerLane][8];
    const long long e_lane = clo + (long long)lane * B::EL;
    const char* lp = p.in + e_lane * B::s;
    if (clo >= E0 && chi <= E1) {
#pragma unroll
      for (int j = 0; j < kBalVecsPerLane; ++j) ld_v8(lp + j * kVecBytes, r[j]);
    } else {  // first / last chunk: partial vectors element by element, outside [E0, E1) the identity
#pragma unroll
      for (int j = 0; j < kBalVecsPerLane; ++j) {
        const long long v0 = e_lane + (long long)j * T::VE;
        if (v0 >= E0 && v0 + T::VE <= E1) {
          ld_v8(lp + j * kVecBytes, r[j]);
        } else {
#pragma unroll
          for (int e = 0; e < T::VE; ++e) {
            const Elem x = (v0 + e >= E0 && v0 + e < E1) ? __ldg((const Elem*)lp + j * T::VE + e) : eid;
            if constexpr (sizeof(Elem) == 4) {
              r[j][e] = *reinterpret_cast<const uint32_t*>(&x);
            } else {
              r[j][2 * e] = (uint32_t)__double2loint(x);
              r[j][2 * e + 1] = (uint32_t)__double2hiint(x);
            }
          }
        }
      }
    }
    // 2. the chunk's offsets slice as chunk-local positions: -1 before the
    // chunk, C at / after its end (the first such entry ends the list)
    int m = 0;
    bool ovf = false;
#pragma unroll 1
    for (long long base = s0;; base += 32) {
      const long long idx = base + lane;
      const long long v = idx <= nseg ? __ldg(p.offsets + idx) : chi;
      const int loc = v < clo ? -1 : (v >= chi ? (int)B::C : (int)(v - clo));
      const unsigned stop = __ballot_sync(0xffffffffu, loc == (int)B::C);
      const int cnt = stop ? __ffs(stop) : 32;
      if (m + cnt > B::kList) {
        ovf = true;
        break;
      }
      if (lane < cnt) list[m + lane] = (short)loc;
      m += cnt;
      if (stop) break;
    }
    __syncwarp();
    if (ovf) {
      bal_chunk_walk<T>(p, c, clo, chi, E0, E1, s0, lane);
      __syncwarp();
      continue;
    }
    // 3. the lane's boundaries as a bit mask (bit e: a segment starts at element e)
    const int a0 = lane * B::EL;
    int i0 = 0;
    {
      int hi_i = m - 1;  // list[m - 1] == C > a0
      while (i0 < hi_i) {
        const int mid = (i0 + hi_i) >> 1;
        if (list[mid] < a0) i0 = mid + 1; else hi_i = mid;
      }
    }
    unsigned long long mask = 0;
#pragma unroll 1
    for (int j = i0; list[j] < a0 + B::EL; ++j) mask |= 1ull << (list[j] - a0);
    const unsigned fb = __ballot_sync(0xffffffffu, mask != 0ull);
    if (fb == 0u) {  // no boundary in the chunk: plain vector-tree fold
      Part<T> acc[T::NA];
      init_parts<T>(acc);
      uint32_t aux = 0;
#pragma unroll
      for (int j = 0; j < kBalVecsPerLane; ++j) fold_vec<T>(acc, aux, r[j], j);
      const Acc w = T::warp(thread_result<T>(acc, aux));
      if (lane == 0) {
        ((Grid*)p.b.first_val)[c] = T::to_grid(w);
        ((Grid*)p.b.last_val)[c] = T::to_grid(w);
        p.b.flags[c] = 0u;
        p.b.last_seg[c] = 0xFFFFFFFFu;
      }
      __syncwarp();
      continue;
    }
    // 4. fold element by element, closing a piece at every boundary
    Part<T> a = PartOf<T>::ident();
    uint32_t aux = 0;
    int np = 0;
#pragma unroll
    for (int e = 0; e < B::EL; ++e) {  // fully unrolled: constant register indices and shifts
      if ((mask >> e) & 1ull) {
        pieces[np * 32 + lane] = T::finish(PartOf<T>::to_acc(a), aux);
        ++np;
        a = PartOf<T>::ident();
        aux = 0;
      }
      bal_fold1<T>(a, aux, bal_elem<T>(r, e));
    }
    const Acc tail = T::finish(PartOf<T>::to_acc(a), aux);
    // 5. segmented inclusive scan over the lanes: a lane with a boundary
    // restarts the running value with its last piece
    const bool f = mask != 0ull;
    Acc x = tail;
    bool ff = f;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const Acc y = shfl_up_v(x, d);
      const bool fy = __shfl_up_sync(0xffffffffu, ff, d);
      if (lane >= d) {
        if (!ff) x = T::comb(y, x);
        ff = ff || fy;
      }
    }
    const Acc carry = shfl_up_v(x, 1);
    __syncwarp();
    if (f) {
      const Acc head = pieces[lane];
      const Acc close = lane > 0 ? T::comb(carry, head) : head;
      if (fb & ((1u << lane) - 1u)) {  // the segment holding element a0 - 1 closes here
        bal_store<T>(p, (long long)s0 + i0 - 1, T::to_grid(close));
      } else {                          // the chunk's first boundary: the incoming segment's piece
        ((Grid*)p.b.first_val)[c] = T::to_grid(close);
      }
      int j = i0;
#pragma unroll 1
      for (int k = 1; k < np; ++k) {  // segments that start and end in this lane
        const int o = list[j];
        while (list[j + 1] == o) ++j;
        bal_store<T>(p, (long long)s0 + j, T::to_grid(pieces[k * 32 + lane]));
        ++j;
      }
    }
    if (lane == 31) {
      const long long ls = (long long)s0 + m - 2;  // the segment open at the chunk's end
      ((Grid*)p.b.last_val)[c] = T::to_grid(x);
      p.b.flags[c] = 1u;
      p.b.last_seg[c] = ls < nseg ? (unsigned)ls : 0xFFFFFFFFu;
    }
    __syncwarp();  // pieces / list are rewritten for the next chunk
  }
  pdl_trigger();
}

template <int DT, int OP>
__global__ void __launch_bounds__(256) k_segbal_fix(const SegParams p) {
  using T = Tr<DT, OP>;
  using B = Bal<T>;
  using Grid = typename T::Grid;
  pdl_wait();
  const long long nseg = p.nseg;
  const long long E0 = __ldg(p.offsets), E1 = __ldg(p.offsets + nseg);
  const unsigned nonmono = *(volatile unsigned*)p.b.hdr;
  const long long P0 = bal_origin<B::s>(p.in, E0);
  const long long nchunks = E1 > E0 ? (E1 - P0 + B::C - 1) / B::C : 0;
  const int lane = threadIdx.x & 31;
  if (!nonmono && nchunks <= (long long)kBalChunks) {
    const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
    const Grid* fv = (const Grid*)p.b.first_val;
#pragma unroll 1
    for (long long c = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); c < nchunks; c += nw) {
      const unsigned ls = __ldcg(p.b.last_seg + c);
      if (!__ldcg(p.b.flags + c) || ls == 0xFFFFFFFFu) continue;  // warp-uniform
      Grid x = __ldcg((const Grid*)p.b.last_val + c);
#pragma unroll 1
      for (long long b0 = c + 1;; b0 += 32) {
        const long long k = b0 + lane;
        Grid v = T::gident();
        unsigned kf = 1u;
        if (k < nchunks) {
          v = __ldcg(fv + k);
          kf = __ldcg(p.b.flags + k);
        }
        const unsigned bal = __ballot_sync(0xffffffffu, kf != 0u);
        const int stop = bal ? __ffs(bal) - 1 : 32;
        if (lane > stop) v = T::gident();
        x = T::gcomb(x, T::gwarp(v));
        if (bal) break;
      }
      if (lane == 0) seg_store<T>(p, ls, x);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && ticket_acq_rel(p.b.hdr + 1) == gridDim.x - 1) {
    p.b.hdr[0] = 0u;
    p.b.hdr[1] = 0u;
  }
  pdl_trigger();
}

template <class K>
cudaError_t bal_launch(K kernel, long long grid, int block, size_t smem, const SegParams& p, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kernel, p);
}

template <int DT, int OP>
cudaError_t launch_segbal_op(const SegParams& p, int sms, cudaStream_t s) {
  using B = Bal<Tr<DT, OP>>;
  constexpr size_t smem = (size_t)kBalWarps * B::kWarpSmem;
  static int per_sm = 0;
  if (per_sm == 0) {
    cudaError_t e = cudaFuncSetAttribute(k_segbal<DT, OP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessorWithFlags(&nb, k_segbal<DT, OP>, kBalWarps * 32, smem, 0) !=
            cudaSuccess || nb < 1)
      nb = 1;
    per_sm = nb;
  }
  cudaError_t e = bal_launch(k_segbal_scan<DT, OP>, (p.nseg + 255) / 256, 256, 0, p, s);
  if (e != cudaSuccess) return e;
  e = bal_launch(k_segbal<DT, OP>, (long long)sms * per_sm, kBalWarps * 32, smem, p, s);
  if (e != cudaSuccess) return e;
  return bal_launch(k_segbal_fix<DT, OP>, (long long)sms * 4, 256, 0, p, s);
}

template <int DT>
cudaError_t launch_segbal_dt(int op, const SegParams& p, cudaStream_t s) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  switch (op) {
    case OP_SUM: return launch_segbal_op<DT, OP_SUM>(p, sms, s);
    case OP_MIN: return launch_segbal_op<DT, OP_MIN>(p, sms, s);
    case OP_MAX: return launch_segbal_op<DT, OP_MAX>(p, sms, s);
    case OP_SUMACC:
      if constexpr (DT != DT_I32) return launch_segbal_op<DT, OP_SUMACC>(p, sms, s);
      break;
  }
  return cudaErrorInvalidValue;
}

}  // namespace rb
