// reduce_segbal.cuh -- element-balanced segmented reduction of an offsets
// array (the variable-length case).
//
// reduce_segmented's group kernels give every segment to one group, so the
// time a group spends depends on the lengths it draws: with power-law lengths
// the grid waits for the few groups that drew long segments, and each short
// segment costs a chain of dependent loads (offsets -> data -> store).  Here
// the ELEMENTS are split evenly instead: the flat range [offsets[0],
// offsets[nseg]) is cut into 4 KB chunks on 32-byte boundaries and one warp
// reduces one chunk whatever the segments inside it look like -- the
// partition is by data, as the paper's tiled distribution of a single array
// (Fig. 1(b)), with segment boundaries carried inside it.
//
//   k_segbal_scan : a one-wave grid striding over the segments: the identity
//                   for empty segments,
//                   a flag if the offsets are not monotone (then the chunk
//                   kernel falls back to one warp per segment), and for every
//                   chunk range the segment holding its first element.
//   k_segbal      : a one-wave grid; warp w owns a contiguous range of chunks
//                   and carries the segment still open from one chunk to the
//                   next.  Per chunk, lane l owns the chunk's 128 bytes
//                   [128 l, 128 l + 128) (four 32-byte loads, issued as soon
//                   as the previous chunk's fold has consumed its data).  The
//                   chunk's slice of the offsets array (its first 64 entries
//                   prefetched) is copied into shared memory as chunk-local
//                   positions; each lane turns the boundaries in its range
//                   into a bit mask, folds its elements in order, closing a
//                   piece at every set bit (the piece a boundary at chunk
//                   position e closes goes to shared slot e).  A segmented
//                   scan over the 32 lanes (5 shuffle steps, fixed order)
//                   joins the pieces of segments that cross lanes.  Segments
//                   that start and end in the chunk are then written in list
//                   order, 32 consecutive outputs per store instruction (the
//                   value of [list[j], list[j+1]) is slot list[j+1]).  A
//                   chunk without boundaries folds with the plain
//                   vector tree.  The range leaves its first piece (the
//                   segment open at its start) and its last (the segment
//                   open at its end) for the fix-up.
//   k_segbal_fix  : one warp per range whose last piece opens a segment: joins
//                   it with the first pieces of the following ranges up to the
//                   range where the segment closes (32 ranges per step, fixed
//                   order), writes out[segment], and the last block resets the
//                   call's flags.
// Chunk size: 4 KB (4 vectors per lane, 96 registers, 20 resident warps per
// SM) measured 15-17 % faster than 8 KB (128 registers, 16 warps): the chunk
// kernel is bound by its per-chunk instruction chain, so resident warps beat
// bytes per warp (profiles/r01_segbal_ab.txt).
// Values never touch atomics and every combine order depends only on the
// offsets: deterministic.  Chunk geometry depends only on the input address
// modulo 32 and offsets[0].
#pragma once
#include <climits>
#include <cstdlib>
#include "reduce_segmented.cuh"

namespace rb {

// Launch shape (A/B hooks: REDUCE_B200_NVCC_FLAGS="-DRB_SEGBAL_VPL=4 ...").
#ifndef RB_SEGBAL_VPL
#define RB_SEGBAL_VPL 4
#endif
#ifndef RB_SEGBAL_MINB
#define RB_SEGBAL_MINB 5
#endif
#ifndef RB_SEGBAL_SPLIT
#define RB_SEGBAL_SPLIT 1
#endif
#ifndef RB_SEGBAL_WARPS
#define RB_SEGBAL_WARPS 4
#endif
constexpr int kBalWarps = RB_SEGBAL_WARPS;      // warps per block of k_segbal
// resident blocks asked of ptxas: 5 (96 registers, 20 warps per SM) for the
// 4-byte plain ops; fp64 and accurate sums need more registers (4 blocks)
constexpr int bal_min_blocks(int dt, int op) { return (dt != 2 && op != 3) ? RB_SEGBAL_MINB : 4; }
constexpr int kBalVecsPerLane = RB_SEGBAL_VPL;  // 32-byte vectors per lane per chunk (128 contiguous bytes)

template <class T>
struct Bal {
  using Acc = typename T::Acc;
  static constexpr int s = sizeof(typename T::Elem);
  static constexpr int EL = kBalVecsPerLane * T::VE;  // elements per lane (32 or 16)
  static constexpr long long C = 32LL * EL;           // elements per chunk (32 lanes x kBalVecsPerLane x 32 B = 4 KB)
  static constexpr int kList = (int)C + 64;           // offsets entries kept in shared memory
  static constexpr size_t kPieceBytes = (size_t)EL * 32 * sizeof(Acc);
  static constexpr size_t kListBytes = ((size_t)kList * 2 + 15) / 16 * 16;
  static constexpr size_t kLaneBytes = 32 * 4;  // per lane: boundary mask word
  static constexpr size_t kWarpSmem = kPieceBytes + kListBytes + kLaneBytes;
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

// element e of a lane's vectors (e is a constant after unrolling)
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

// The chunks are split into contiguous ranges, one per warp of k_segbal's
// grid: range w = [cb(w), cb(w + 1)), cb(w) = w*per + min(w, rem).
struct BalRanges {
  long long per, rem;
  __device__ BalRanges(long long nchunks, long long nranges) : per(nchunks / nranges), rem(nchunks % nranges) {}
  __device__ long long begin(long long w) const { return w * per + (w < rem ? w : rem); }
  // the first range starting at or after chunk c
  __device__ long long first_at(long long c) const {
    if (per == 0) return c;
    const long long t = rem * (per + 1);
    return c <= t ? (c + per) / (per + 1) : rem + (c - t + per - 1) / per;
  }
};

// BalRanges in 32-bit arithmetic for the scan (chunk counts below 2^31: inline
// 32-bit divisions instead of the 64-bit division routine; the per-segment form
// of round 1 diverged on that arithmetic, 4.3 of the scan's 7.4 us)
struct BalRanges32 {
  unsigned per, rem, t;
  __device__ BalRanges32(unsigned nchunks, unsigned nranges)
      : per(nchunks / nranges), rem(nchunks % nranges), t(rem * (per + 1u)) {}
  __device__ unsigned begin(unsigned w) const { return w * per + (w < rem ? w : rem); }
  __device__ unsigned first_at(unsigned c) const {
    if (per == 0) return c;
    return c <= t ? (c + per) / (per + 1u) : rem + (c - t + per - 1u) / per;
  }
};

template <int DT, int OP, int K>
__global__ void __launch_bounds__(256) k_segbal_scan(const SegParams p) {
  using T = Tr<DT, OP>;
  using B = Bal<T>;
  pdl_wait();
  // one-wave grid striding over the segments (the per-call geometry once per thread)
  const long long E0 = __ldg(p.offsets), E1 = __ldg(p.offsets + p.nseg);
  const long long P0 = bal_origin<B::s>(p.in, E0);
  const long long nchunks = E1 > E0 ? (E1 - P0 + B::C - 1) / B::C : 0;
  const bool narrow = nchunks < (1ll << 31) && p.b.nranges < (1ll << 31);
  // K consecutive segments per thread per step (K from the host: the fewest
  // steps for the grid), their K + 1 offsets loaded before any is used -- the
  // loop is latency-bound, one round trip per step
  const long long nthreads = (long long)gridDim.x * blockDim.x;
#pragma unroll 1
  for (long long i0 = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * K; i0 < p.nseg; i0 += nthreads * K) {
    long long o[K + 1];
#pragma unroll
    for (int j = 0; j <= K; ++j) o[j] = i0 + j <= p.nseg ? __ldg(p.offsets + i0 + j) : LLONG_MAX;
    // the identity for empty segments, the flag for decreasing offsets
#pragma unroll
    for (int j = 0; j < K; ++j) {
      if (i0 + j < p.nseg) {
        if (o[j + 1] < o[j]) atomicOr(p.b.hdr, 1u);
        if (o[j + 1] <= o[j]) seg_store<T>(p, i0 + j, T::gident());
      }
    }
    // start_seg[w] for the ranges whose first chunk starts in this thread's
    // elements [o[0], o[K'])  (chunk 0 starts at E0, chunk c > 0 at P0 + c*C;
    // once per thread, not per segment: the per-segment form diverged on the
    // range arithmetic, 4.3 of the scan's 7.4 us)
    if (nchunks > 0) {
      const long long kv = p.nseg - i0 < K ? p.nseg - i0 : K;  // segments this thread holds
      long long hi = o[0];
#pragma unroll
      for (int j = 1; j <= K; ++j)
        if (j <= kv) hi = o[j];
      const long long lo = o[0];
      const long long c0 = lo <= E0 ? 0 : (long long)((unsigned long long)(lo - P0 + B::C - 1) / B::C);
      long long c1 = hi <= E0 ? 0 : (long long)((unsigned long long)(hi - P0 + B::C - 1) / B::C);
      if (c1 > nchunks) c1 = nchunks;
      if (c0 < c1) {
        auto claim = [&](long long w, long long cs) {
          const long long pos = cs == 0 ? E0 : P0 + cs * B::C;
          // the non-empty segment holding pos: the last j with o[j] <= pos
          int js = 0;
#pragma unroll
          for (int j = 1; j < K; ++j)
            if (j < kv && o[j] <= pos) js = j;
          p.b.start_seg[w] = (unsigned)(i0 + js);
        };
        if (narrow) {
          const BalRanges32 R((unsigned)nchunks, (unsigned)p.b.nranges);
          for (unsigned w = R.first_at((unsigned)c0); w < (unsigned)p.b.nranges && R.begin(w) < (unsigned)c1; ++w)
            claim(w, R.begin(w));
        } else {
          const BalRanges R(nchunks, p.b.nranges);
          for (long long w = R.first_at(c0); w < p.b.nranges && R.begin(w) < c1; ++w) claim(w, R.begin(w));
        }
      }
    }
  }
  pdl_trigger();
}

// What one chunk leaves for the range it belongs to (warp-uniform).
template <class T>
struct BalChunk {
  typename T::Grid first;  // piece of the segment open at the chunk's start (whole chunk if !has_b)
  typename T::Grid last;   // piece of the segment open at its end (if has_b)
  unsigned last_seg;       // that segment (0xFFFFFFFF: none, past the last offset)
  bool has_b;              // a segment boundary lies in the chunk
  long long s_next;        // the segment holding the chunk's last element (next chunk's list start)
};

// The slow path of one chunk (its offsets slice does not fit the shared list:
// thousands of empty segments): walk the segments in global memory, one warp
// fold per piece.  Same outputs as the fast path.
template <class T>
__device__ __forceinline__ BalChunk<T> bal_chunk_walk(const SegParams& p, long long clo, long long chi,
                                                      long long E0, long long E1, long long s0, int lane) {
  const long long nseg = p.nseg;
  const long long vlo = clo > E0 ? clo : E0, vhi = chi < E1 ? chi : E1;
  BalChunk<T> r;
  r.first = r.last = T::gident();
  r.last_seg = 0xFFFFFFFFu;
  long long j = s0;
  bool incoming = __ldg(p.offsets + j) < clo;
  r.has_b = !incoming;
  r.s_next = s0;
  long long pos = vlo;
  while (true) {
    const long long end = __ldg(p.offsets + j + 1);
    const typename T::Acc v = bal_warp_range<T>(p, pos, end < vhi ? end : vhi, lane);
    if (end < chi) {  // segment j closes inside the chunk
      if (incoming) {
        r.first = T::to_grid(v);
        incoming = false;
        r.has_b = true;
      } else if (lane == 0) {
        bal_store<T>(p, j, T::to_grid(v));
      }
      long long i = j + 1;  // the non-empty segment starting at `end`
      while (i < nseg && __ldg(p.offsets + i + 1) == end) ++i;
      j = i;
      pos = end;
      if (j >= nseg) break;
    } else {
      if (incoming) r.first = T::to_grid(v);
      else { r.last = T::to_grid(v); r.last_seg = (unsigned)j; }
      r.s_next = j;
      break;
    }
  }
  return r;
}

template <class V>
__device__ __forceinline__ V shfl_idx_v(V v, int src) { return __shfl_sync(0xffffffffu, v, src); }
__device__ __forceinline__ double2 shfl_idx_v(double2 v, int src) {
  return make_double2(__shfl_sync(0xffffffffu, v.x, src), __shfl_sync(0xffffffffu, v.y, src));
}

// 8 x 32-byte loads of lane `lane` of an interior chunk (all in flight)
template <class T>
__device__ __forceinline__ void bal_load(const char* in, long long clo, int lane, uint32_t (&r)[kBalVecsPerLane][8]) {
  const char* lp = in + (clo + (long long)lane * Bal<T>::EL) * Bal<T>::s;
#pragma unroll
  for (int j = 0; j < kBalVecsPerLane; ++j) ld_v8(lp + j * kVecBytes, r[j]);
}

// the same for the first / last chunk: partial vectors element by element,
// positions outside [E0, E1) hold the identity
template <class T>
__device__ __forceinline__ void bal_load_edge(const char* in, long long clo, long long E0, long long E1, int lane,
                                              uint32_t (&r)[kBalVecsPerLane][8]) {
  using Elem = typename T::Elem;
  const Elem eid = elem_ident<T>();
  const long long e_lane = clo + (long long)lane * Bal<T>::EL;
  const char* lp = in + e_lane * Bal<T>::s;
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

// The segment holding element chi - 1 (next chunk's list start) when the
// chunk's offsets slice overflowed the shared list: scan on from `from`.
__device__ __forceinline__ long long bal_walk_next(const long long* offsets, long long nseg, long long from,
                                                   long long chi, int lane) {
#pragma unroll 1
  for (long long base = from;; base += 32) {
    const long long idx = base + lane;
    const long long v = idx <= nseg ? __ldg(offsets + idx) : LLONG_MAX;
    const unsigned b = __ballot_sync(0xffffffffu, v >= chi);
    if (b) return base + __ffs(b) - 2;
  }
}

template <int DT, int OP>
__global__ void __launch_bounds__(kBalWarps * 32, bal_min_blocks(DT, OP)) k_segbal(const SegParams p) {
  using T = Tr<DT, OP>;
  using B = Bal<T>;
  using Acc = typename T::Acc;
  using Grid = typename T::Grid;
  extern __shared__ __align__(16) unsigned char bal_smem[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  Acc* pieces = reinterpret_cast<Acc*>(bal_smem + wib * B::kWarpSmem);
  short* list = reinterpret_cast<short*>(bal_smem + wib * B::kWarpSmem + B::kPieceBytes);
  unsigned* lmask = reinterpret_cast<unsigned*>(bal_smem + wib * B::kWarpSmem + B::kPieceBytes + B::kListBytes);
  pdl_wait();
  const long long nseg = p.nseg;
  const long long E0 = __ldg(p.offsets), E1 = __ldg(p.offsets + nseg);
  const unsigned nonmono = *(volatile unsigned*)p.b.hdr;
  const long long P0 = bal_origin<B::s>(p.in, E0);
  const long long nchunks = E1 > E0 ? (E1 - P0 + B::C - 1) / B::C : 0;
  const long long gw = (long long)blockIdx.x * kBalWarps + wib, nw = p.b.nranges;
  if (nonmono) {
    // offsets not monotone (overlapping segments): one warp per segment
#pragma unroll 1
    for (long long seg = gw; seg < nseg; seg += nw) {
      const long long lo = __ldg(p.offsets + seg), hi = __ldg(p.offsets + seg + 1);
      if (hi <= lo) continue;
      const Acc w = bal_warp_range<T>(p, lo, hi, lane);
      if (lane == 0) seg_store<T>(p, seg, T::to_grid(w));
    }
    if (lane == 0) {  // no range pieces: the fix-up joins nothing
      p.b.flags[gw] = 0u;
      p.b.last_seg[gw] = 0xFFFFFFFFu;
    }
    pdl_trigger();
    return;
  }
  const BalRanges R(nchunks, nw);
  const long long cb = R.begin(gw), ce = R.begin(gw + 1);
  // the range's carry: the piece of the segment open at the range's start
  // (until the range's first boundary), then the segment opened last
  Grid rfirst = T::gident(), carry = T::gident();
  bool seen = false;
  unsigned carry_seg = 0xFFFFFFFFu;
  auto absorb = [&](const BalChunk<T>& k) {
    if (!k.has_b) {
      if (seen) carry = T::gcomb(carry, k.first); else rfirst = T::gcomb(rfirst, k.first);
    } else {
      if (seen) {
        if (lane == 0 && carry_seg != 0xFFFFFFFFu) seg_store<T>(p, carry_seg, T::gcomb(carry, k.first));
      } else {
        rfirst = T::gcomb(rfirst, k.first);
        seen = true;
      }
      carry = k.last;
      carry_seg = k.last_seg;
    }
  };
  auto interior = [&](long long c) {
    const long long clo = P0 + c * B::C;
    return clo >= E0 && clo + B::C <= E1;
  };
  // list start of the current chunk and its first two batches of offsets
  // (prefetched while the previous chunk is folded)
  long long s0 = 0, vfirst = 0, vsecond = 0;
  auto prefetch_list = [&](long long s) {
    vfirst = s + lane <= nseg ? __ldg(p.offsets + s + lane) : LLONG_MAX;
    vsecond = s + 32 + lane <= nseg ? __ldg(p.offsets + s + 32 + lane) : LLONG_MAX;
  };
  // the chunk's data: loaded into `cur` as soon as the previous chunk's fold
  // has consumed it, so the loads fly during that chunk's scan / emission and
  // this chunk's offsets processing
  uint32_t cur[kBalVecsPerLane][8];
  auto load_data = [&](long long c) {
    if (c >= ce) return;
    const long long clo = P0 + c * B::C;
    if (interior(c)) bal_load<T>(p.in, clo, lane, cur);
    else bal_load_edge<T>(p.in, clo, E0, E1, lane, cur);
  };
  auto body = [&](long long c) {
    const long long clo = P0 + c * B::C, chi = clo + B::C;
    // the chunk's offsets slice as chunk-local positions: -1 before the
    // chunk, C at / after its end (the first such entry ends the list)
    int m = 0;
    bool ovf = false;
    long long v = vfirst;
    // per lane: the bits of the boundaries in its elements and how many list
    // entries fall there, set with shared atomics as the list is built (no
    // per-lane search of the list afterwards)
    lmask[lane] = 0u;
    __syncwarp();
    // batches past the two prefetched ones are loaded four at a time (chunks
    // of very short segments need dozens: one round trip per four, not per one)
    long long q0 = 0, q1 = 0, q2 = 0, q3 = 0;
    int nq = 0;
#pragma unroll 1
    for (long long base = s0;;) {
      const int loc = v < clo ? -1 : (v >= chi ? (int)B::C : (int)(v - clo));
      const unsigned stop = __ballot_sync(0xffffffffu, loc == (int)B::C);
      const int cnt = stop ? __ffs(stop) : 32;
      if (m + cnt > B::kList) {
        ovf = true;
        break;
      }
      if (lane < cnt) {
        list[m + lane] = (short)loc;
        if (loc >= 0 && loc < (int)B::C) atomicOr(lmask + loc / B::EL, 1u << (loc % B::EL));
      }
      m += cnt;
      if (stop) break;
      base += 32;
      if (base == s0 + 32) {
        v = vsecond;
      } else {
        if (nq == 0) {
          q0 = base + lane <= nseg ? __ldg(p.offsets + base + lane) : LLONG_MAX;
          q1 = base + 32 + lane <= nseg ? __ldg(p.offsets + base + 32 + lane) : LLONG_MAX;
          q2 = base + 64 + lane <= nseg ? __ldg(p.offsets + base + 64 + lane) : LLONG_MAX;
          q3 = base + 96 + lane <= nseg ? __ldg(p.offsets + base + 96 + lane) : LLONG_MAX;
          nq = 4;
        }
        v = q0;
        q0 = q1;
        q1 = q2;
        q2 = q3;
        --nq;
      }
    }
    __syncwarp();
    BalChunk<T> k;
    k.s_next = s0 + m - 2;
    if (ovf) k.s_next = bal_walk_next(p.offsets, nseg, s0 + m, chi, lane);
    if (c + 1 < ce) prefetch_list(k.s_next);  // the next chunk's offsets, while this one folds
    unsigned long long mask = 0;
    unsigned fb = 0;
    Acc tv = T::ident();  // the lane's value (no boundary in the chunk) or its last piece
    // an interior next chunk is loaded in two halves, the first as soon as the
    // fold has consumed the first half of `cur` (RB_SEGBAL_SPLIT; power-law
    // 60.4 -> 57.6 us; each vector as soon as it is consumed: slower,
    // profiles/r02_segbal_split_ab.txt, profiles/r02_segbal_split2_ab.txt)
    const bool split = RB_SEGBAL_SPLIT && !ovf && c + 1 < ce && interior(c + 1);
    const char* lpn = p.in + ((P0 + (c + 1) * B::C) + (long long)lane * B::EL) * B::s;
    auto load_half = [&](int h) {
#pragma unroll
      for (int j = h * kBalVecsPerLane / 2; j < (h + 1) * kBalVecsPerLane / 2; ++j) ld_v8(lpn + j * kVecBytes, cur[j]);
    };
    if (!ovf) {
      // the lane's boundaries as a bit mask (bit e: a segment starts at element e)
      mask = lmask[lane];
      fb = __ballot_sync(0xffffffffu, mask != 0ull);
      if (fb == 0u) {  // no boundary in the chunk: plain vector-tree fold
        Part<T> acc[T::NA];
        init_parts<T>(acc);
        uint32_t aux = 0;
#pragma unroll
        for (int j = 0; j < kBalVecsPerLane; ++j) {
          fold_vec<T>(acc, aux, cur[j], j);
          if (j == kBalVecsPerLane / 2 - 1 && split) load_half(0);
        }
        tv = thread_result<T>(acc, aux);
      } else {
        // fold element by element; the piece that a boundary at element e
        // closes goes to slot e of the lane (pieces[e * 32 + lane]: a constant
        // address per element, bank = lane)
        Part<T> a = PartOf<T>::ident();
        uint32_t aux = 0;
#pragma unroll
        for (int e = 0; e < B::EL; ++e) {  // fully unrolled: constant register indices and shifts
          if (e == B::EL / 2 && split) load_half(0);  // the first half of `cur` is consumed
          if ((mask >> e) & 1ull) {
            pieces[e * 32 + lane] = T::finish(PartOf<T>::to_acc(a), aux);
            a = PartOf<T>::ident();
            aux = 0;
          }
          bal_fold1<T>(a, aux, bal_elem<T>(cur, e));
        }
        tv = T::finish(PartOf<T>::to_acc(a), aux);
      }
    }
    if (split) load_half(1);
    else load_data(c + 1);  // `cur` is consumed: the next chunk's loads fly from here  // `cur` is consumed: the next chunk's loads fly from here
    if (ovf) {
      const long long sn = k.s_next;
      k = bal_chunk_walk<T>(p, clo, chi, E0, E1, s0, lane);
      k.s_next = sn;
    } else if (fb == 0u) {
      k.first = T::to_grid(T::warp(tv));
      k.has_b = false;
    } else {
      {
        // segmented inclusive scan over the lanes: a lane with a boundary
        // restarts the running value with its last piece
        const bool f = mask != 0ull;
        Acc x = tv;
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
        const Acc carry_in = shfl_up_v(x, 1);
        Grid firstv = T::gident();
        if (f) {
          // the lane's first piece closes the segment open at its start
          const int e1 = __ffsll((long long)mask) - 1;
          const Acc head = pieces[e1 * 32 + lane];
          const Acc close = lane > 0 ? T::comb(carry_in, head) : head;
          if (fb & ((1u << lane) - 1u)) pieces[e1 * 32 + lane] = close;  // opened in this chunk
          else firstv = T::to_grid(close);  // the chunk's first boundary: the incoming segment
        }
        __syncwarp();
        // every segment that starts and ends in the chunk, in list order (one
        // coalesced store per 32): segment s0 + j is [list[j], list[j + 1]);
        // its value is the piece closed at list[j + 1] (empty segments keep
        // the identity the scan kernel wrote)
        const int jA = list[0] < 0 ? 1 : 0;
#pragma unroll 1
        for (int j = jA + lane; j < m - 2; j += 32) {
          const int lo = list[j], hi = list[j + 1];
          if (lo != hi) bal_store<T>(p, (long long)s0 + j, T::to_grid(pieces[(hi % B::EL) * 32 + hi / B::EL]));
        }
        k.first = shfl_idx_v(firstv, __ffs(fb) - 1);
        k.last = shfl_idx_v(T::to_grid(x), 31);
        const long long ls = (long long)s0 + m - 2;  // the segment open at the chunk's end
        k.last_seg = ls < nseg ? (unsigned)ls : 0xFFFFFFFFu;
        k.has_b = true;
      }
    }
    __syncwarp();  // pieces / list are rewritten for the next chunk
    absorb(k);
    s0 = k.s_next;
  };
  if (cb < ce) {
    s0 = __ldcg(p.b.start_seg + gw);
    prefetch_list(s0);
    load_data(cb);
#pragma unroll 1
    for (long long c = cb; c < ce; ++c) body(c);
  }
  if (lane == 0) {  // the range's pieces for the fix-up
    ((Grid*)p.b.first_val)[gw] = rfirst;
    ((Grid*)p.b.last_val)[gw] = seen ? carry : rfirst;
    p.b.flags[gw] = seen ? 1u : 0u;
    p.b.last_seg[gw] = seen ? carry_seg : 0xFFFFFFFFu;
  }
  pdl_trigger();
}

// One warp per range whose last piece opens a segment: joins it with the
// first pieces of the following ranges up to the one where the segment closes
// (32 ranges per step, fixed order).  Block 0 clears the call's non-monotone
// flag: every reader (the chunk kernel) has completed, and the chunk kernel's
// fallback leaves no open range pieces, so this kernel never needs the flag
// (round 2: no end-of-call ticket, fix 3.7 -> 2.7 us,
// profiles/r02_segbal_fix_noticket_ab.txt).
template <int DT, int OP>
__global__ void __launch_bounds__(256) k_segbal_fix(const SegParams p) {
  using T = Tr<DT, OP>;
  using Grid = typename T::Grid;
  pdl_wait();
  if (blockIdx.x == 0 && threadIdx.x == 0) p.b.hdr[0] = 0u;
  const long long nr = p.b.nranges;
  const int lane = threadIdx.x & 31;
  {
    const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
    const Grid* fv = (const Grid*)p.b.first_val;
#pragma unroll 1
    for (long long c = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); c < nr; c += nw) {
      // this range's words and the first batch of the following ranges' in
      // one round of loads (most segments close in the next range)
      const unsigned ls = __ldcg(p.b.last_seg + c), fc = __ldcg(p.b.flags + c);
      Grid x = __ldcg((const Grid*)p.b.last_val + c);
      long long k = c + 1 + lane;
      Grid v = T::gident();
      unsigned kf = 1u;
      if (k < nr) {
        v = __ldcg(fv + k);
        kf = __ldcg(p.b.flags + k);
      }
      if (!fc || ls == 0xFFFFFFFFu) continue;  // warp-uniform
#pragma unroll 1
      for (long long b0 = c + 1;; b0 += 32) {
        if (b0 != c + 1) {
          k = b0 + lane;
          v = T::gident();
          kf = 1u;
          if (k < nr) {
            v = __ldcg(fv + k);
            kf = __ldcg(p.b.flags + k);
          }
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

// Measurement only (tools/probes/segbal_split.py): REDUCE_SEGBAL_ONLY=scan|main|fix
// launches just that kernel of the three, reusing what the previous full call
// left in the workspace (same inputs: same values), to time each in a graph.
// (read on every call once it was set at the first call: the probe switches it)
inline int segbal_only() {
  static const bool probing = std::getenv("REDUCE_SEGBAL_ONLY") != nullptr;
  if (!probing) return 0;
  const char* e = std::getenv("REDUCE_SEGBAL_ONLY");
  return !e ? 0 : (e[0] == 's' ? 1 : (e[0] == 'm' ? 2 : (e[0] == 'f' ? 3 : 0)));
}

template <int DT, int OP>
cudaError_t launch_segbal_op(const SegParams& p0, int sms, cudaStream_t s) {
  using B = Bal<Tr<DT, OP>>;
  constexpr size_t smem = (size_t)kBalWarps * B::kWarpSmem;
  cudaError_t e = opt_in_smem((const void*)k_segbal<DT, OP>, (int)smem);
  if (e != cudaSuccess) return e;
  const int per_sm = blocks_per_sm((const void*)k_segbal<DT, OP>, kBalWarps * 32, smem);
  SegParams p = p0;
  long long grid = (long long)sms * per_sm;  // one wave: every warp owns one contiguous chunk range
  if (grid * kBalWarps > (long long)kBalRanges) grid = kBalRanges / kBalWarps;
  p.b.nranges = grid * kBalWarps;
  // the scan: one step per thread where the grid allows (K segments each)
  const long long full = (long long)sms * 8 * 256;
  const int K = p.nseg <= full ? 1 : (p.nseg <= 4 * full ? 4 : 8);
  long long sgrid = (p.nseg + 256ll * K - 1) / (256ll * K);
  if (sgrid > (long long)sms * 8) sgrid = (long long)sms * 8;
  const int only = segbal_only();
  if (only == 0 || only == 1) {
    e = K == 1 ? bal_launch(k_segbal_scan<DT, OP, 1>, sgrid, 256, 0, p, s)
               : (K == 4 ? bal_launch(k_segbal_scan<DT, OP, 4>, sgrid, 256, 0, p, s)
                         : bal_launch(k_segbal_scan<DT, OP, 8>, sgrid, 256, 0, p, s));
    if (e != cudaSuccess) return e;
  }
  if (only == 0 || only == 2) {
    e = bal_launch(k_segbal<DT, OP>, grid, kBalWarps * 32, smem, p, s);
    if (e != cudaSuccess) return e;
  }
  if (only == 0 || only == 3) return bal_launch(k_segbal_fix<DT, OP>, (p.b.nranges + 7) / 8, 256, 0, p, s);
  return cudaSuccess;
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
