// reduce_segmented.cuh -- many independent reductions in one call (SURVEY
// section 8(f) N1: batched / segmented reduction).
//
// Segment i is in[lo_i, hi_i) with lo_i = offsets[i], hi_i = offsets[i+1]
// (device int64 array of num_segments + 1 entries), or lo_i = i * seg_len for
// uniform batches (offsets == NULL); out[i] receives its result.  The paper's
// small-array winners assign one warp or one block per
// partition with no global atomics; here the group size is chosen from the
// segment length (host side, reduce_api.cpp):
//   kGroup == 1     : one thread per segment (rows of a few vectors);
//   kGroup == 8     : 8 lanes per segment (4 segments per warp), shuffles;
//   kGroup == 32    : one warp per segment, warp combine only (redux / shuffles);
//   kGroup == 0     : one block per segment, block combine "Vs".
// Each segment gets its own head / 32-byte-aligned body / tail split, so any
// element-aligned offset works.
//
// Load balance.  A group reduces the first round of its segment (one vector
// per lane, plus head and tail); a segment with more than kLongVecs vectors
// left is not finished by the group: the group's partial goes into the
// stream's long-segment queue with the rest of the segment cut into chunks of
// kChunkVecs vectors (k_segmented, leader thread: integer atomics reserve the
// slots), whole blocks of a persistent grid reduce the chunks (k_seg_chunks),
// and one warp per long segment combines its partials in chunk order
// (k_seg_finish, which also resets the queue).  So one huge segment among
// millions of short ones is spread over the GPU instead of one warp.  Values
// never touch atomics and every combine is in a fixed order: deterministic.
#pragma once
#include "reduce_kernels.cuh"

namespace rb {

// A segment in[lo, hi) split into a head (< 32 B, up to the first 32-byte
// boundary), `nvec` aligned 32-byte vectors and a tail (< 32 B).
struct SegGeo {
  const char* p;     // first element
  const char* body;  // first aligned vector
  long long nvec;
  int head, tail;    // elements
};

template <class T>
__device__ __forceinline__ SegGeo seg_geo(const char* base, long long lo, long long hi) {
  constexpr int s = sizeof(typename T::Elem);
  SegGeo g;
  const long long n = hi > lo ? hi - lo : 0;
  g.p = base + lo * s;
  const unsigned mis = (unsigned)((uintptr_t)g.p & 31u);
  long long head = mis ? (long long)((32u - mis) / s) : 0;
  if (head > n) head = n;
  g.head = (int)head;
  g.body = g.p + head * s;
  g.nvec = (n - head) / T::VE;
  g.tail = (int)((n - head) % T::VE);
  return g;
}

// Fold vectors v0, v0 + lanes, ... < nvec of a segment body: full rounds of U
// loads in flight, then the last (< U) vectors either in one predicated round
// (kTail: more loads in flight, more registers) or one at a time.  B200
// (tools/probes/seg_tail_ab.sh): the predicated round wins for rows >= 2 KB
// and for accurate sums, one at a time (64 registers) for short rows.
template <class T, int U, bool kTail = false>
__device__ __forceinline__ void fold_body(Part<T> (&a)[T::NA], uint32_t& aux, const char* body,
                                          long long v0, long long nvec, int lanes) {
  long long v = v0;
#pragma unroll 1
  for (; v + (long long)(U - 1) * lanes < nvec; v += (long long)U * lanes) {
    uint32_t r[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) ld_v8(body + (v + (long long)u * lanes) * kVecBytes, r[u]);
#pragma unroll
    for (int u = 0; u < U; ++u) fold_vec<T>(a, aux, r[u], u);
  }
  if constexpr (kTail) {
    if (v < nvec) {
      uint32_t r[U - 1][8];
#pragma unroll
      for (int u = 0; u < U - 1; ++u)
        if (v + (long long)u * lanes < nvec) ld_v8(body + (v + (long long)u * lanes) * kVecBytes, r[u]);
#pragma unroll
      for (int u = 0; u < U - 1; ++u)
        if (v + (long long)u * lanes < nvec) fold_vec<T>(a, aux, r[u], u);
    }
  } else {
#pragma unroll 1
    for (; v < nvec; v += lanes) {
      uint32_t r[8];
      ld_v8(body + v * kVecBytes, r);
      fold_vec<T>(a, aux, r, 0);
    }
  }
}

// Fold in[lo, hi) by `lanes` cooperating threads (this one is `lid`).
template <class T, int U>
__device__ __forceinline__ void fold_range(Part<T> (&a)[T::NA], uint32_t& aux, const char* base,
                                           long long lo, long long hi, int lid, int lanes) {
  using Elem = typename T::Elem;
  if (hi <= lo) return;
  const SegGeo g = seg_geo<T>(base, lo, hi);
  fold_body<T, U>(a, aux, g.body, lid, g.nvec, lanes);
  // head and tail (< 8 elements each) by the first lanes, into two different
  // accumulators (groups may be only 8 lanes wide)
  if (lid < g.head) fold_elem<T>(a[0], aux, __ldg((const Elem*)g.p + lid));
  if (lid < g.tail) fold_elem<T>(a[T::NA - 1], aux, __ldg((const Elem*)(g.body + g.nvec * kVecBytes) + lid));
}

template <class T>
__device__ __forceinline__ void seg_store(const SegParams& p, long long seg, typename T::Grid g) {
  if (p.raw_out) ((typename T::Grid*)p.out)[seg] = g;
  else T::finalize(g, (char*)p.out + seg * (long long)sizeof(typename T::Elem));
}

template <class T>
__device__ __forceinline__ void seg_bounds(const SegParams& p, long long seg, long long& lo, long long& hi) {
  lo = hi = 0;
  if (seg < p.nseg) {
    if (p.offsets) {
      lo = __ldg(p.offsets + seg);
      hi = __ldg(p.offsets + seg + 1);
    } else {
      lo = seg * p.seg_len;
      hi = lo + p.seg_len;
    }
  }
}

// Segments a small group keeps in flight: the first-round loads of kSegPipe
// segments are issued before any of them is folded (B200 A/B, tools/seg_bench.py:
// 2 beats 1 on short rows; 4 needs 128 registers and loses).
#ifndef RB_SEG_PIPE
#define RB_SEG_PIPE 2
#endif
constexpr int kSegPipe = RB_SEG_PIPE;

// Vectors left after a group's first round above which a segment goes to the
// long-segment queue.
template <int kGroup>
__host__ __device__ constexpr long long seg_long_vecs() {
  return kGroup == 1 ? 32 : kGroup == 8 ? 512 : kGroup == 32 ? 2048 : 8192;
}
// Chunks of a queued segment: at least kChunkMinVecs vectors (16 KB, four
// rounds of four loads for the warp that reduces one), at most kMaxChunks per
// segment (one huge segment still spreads over thousands of warps).
constexpr long long kChunkMinVecs = 512;
constexpr long long kMaxChunks = 4096;
constexpr unsigned kNoSlot = 0xFFFFFFFFu;

// Chunk geometry of a queued remainder of nv vectors: chunk size and count.
__device__ __forceinline__ void seg_chunks(long long nv, long long& per_v, long long& k) {
  per_v = (nv + kMaxChunks - 1) / kMaxChunks;
  if (per_v < kChunkMinVecs) per_v = kChunkMinVecs;
  k = (nv + per_v - 1) / per_v;
}

// Leader of a group: reserve queue slots for the rest of segment `seg` --
// elements [rem_lo, rem_hi), 32-byte aligned at both ends -- and write its
// chunk items.  Slot `base` is left for the group's own partial (written
// after the group combine), chunks take base+1 .. base+k.  Returns kNoSlot if
// the queue is full: the group then finishes the segment itself.
__device__ __forceinline__ unsigned seg_reserve(unsigned* hdr, long long* items, long long* longs, long long seg,
                                             long long rem_lo, long long rem_hi, int ve) {
  long long per_v, k;
  seg_chunks((rem_hi - rem_lo) / ve, per_v, k);
  const long long per = per_v * ve;
  const unsigned need = (unsigned)(k + 1);
  const unsigned base = atomicAdd(hdr + 0, need);
  if ((unsigned long long)base + need > kSegQItems) {
    // reserved past the end: leave the reachable part of the range empty
    for (unsigned long long i = base; i < kSegQItems; ++i) {
      items[2 * i] = 0;
      items[2 * i + 1] = 0;
    }
    return kNoSlot;
  }
  items[2 * (size_t)base] = 0;  // the group's partial: an empty item
  items[2 * (size_t)base + 1] = 0;
  for (long long c = 0; c < k; ++c) {
    const long long lo = rem_lo + c * per;
    items[2 * (base + 1 + c)] = lo;
    items[2 * (base + 1 + c) + 1] = lo + per < rem_hi ? lo + per : rem_hi;
  }
  const unsigned j = atomicAdd(hdr + 1, 1u);  // < kSegQLongs: every long segment holds >= 2 items
  longs[3 * (size_t)j] = seg;
  longs[3 * (size_t)j + 1] = base;
  longs[3 * (size_t)j + 2] = k + 1;
  return base;
}

// Warp-collective seg_reserve (every lane of the warp calls it; `want` lanes
// queue their segment): one atomic per warp on each queue counter instead of
// one per segment -- with many long segments the two same-address counters
// were the bottleneck.
__device__ __forceinline__ unsigned seg_reserve_warp(const SegParams& p, bool want, long long seg, long long rem_lo,
                                                     long long rem_hi, int ve, int lane) {
  long long per_v = 0, k = 0;
  unsigned need = 0;
  if (want) {
    seg_chunks((rem_hi - rem_lo) / ve, per_v, k);
    need = (unsigned)(k + 1);
  }
  unsigned incl = need;  // inclusive prefix of the warp's needs
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned t = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += t;
  }
  const unsigned total = __shfl_sync(0xffffffffu, incl, 31);
  if (total == 0) return kNoSlot;
  unsigned wbase = 0;
  if (lane == 0) wbase = atomicAdd(p.q.hdr + 0, total);
  wbase = __shfl_sync(0xffffffffu, wbase, 0);
  const unsigned long long base = (unsigned long long)wbase + incl - need;
  const bool fits = want && base + need <= kSegQItems;
  if (want && !fits) {  // past the end: leave the reachable part of the range empty
    for (unsigned long long i = base; i < kSegQItems && i < base + need; ++i) {
      p.q.items[2 * i] = 0;
      p.q.items[2 * i + 1] = 0;
    }
  }
  const unsigned fit_mask = __ballot_sync(0xffffffffu, fits);
  unsigned lbase = 0;
  if (lane == 0 && fit_mask) lbase = atomicAdd(p.q.hdr + 1, (unsigned)__popc(fit_mask));
  lbase = __shfl_sync(0xffffffffu, lbase, 0);
  if (!fits) return kNoSlot;
  const long long per = per_v * ve;
  p.q.items[2 * base] = 0;  // the group's partial: an empty item
  p.q.items[2 * base + 1] = 0;
  for (long long c = 0; c < k; ++c) {
    const long long lo = rem_lo + c * per;
    p.q.items[2 * (base + 1 + c)] = lo;
    p.q.items[2 * (base + 1 + c) + 1] = lo + per < rem_hi ? lo + per : rem_hi;
  }
  const unsigned j = lbase + __popc(fit_mask & ((1u << lane) - 1u));
  p.q.longs[3 * (size_t)j] = seg;
  p.q.longs[3 * (size_t)j + 1] = (long long)base;
  p.q.longs[3 * (size_t)j + 2] = k + 1;
  return (unsigned)base;
}

// kGroup = 1, 8 or 32 lanes per segment (32 / kGroup segments per warp at a
// time, kSegPipe of them in flight); kGroup = 0: one block per segment.  The
// grid is persistent (one wave) and groups stride over the segments, so
// millions of tiny segments do not pay one CTA launch each.
template <int DT, int OP, int kGroup, bool kTail>
__global__ void __launch_bounds__(512) k_segmented(const SegParams p) {
  using T = Tr<DT, OP>;
  using Acc = typename T::Acc;
  using Elem = typename T::Elem;
  using Grid = typename T::Grid;
  constexpr long long kLong = seg_long_vecs<kGroup>();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  if constexpr (kGroup > 0) {
    const long long groups_per_block = blockDim.x / kGroup;
    const long long first = (long long)blockIdx.x * groups_per_block + threadIdx.x / kGroup;
    const long long step = (long long)gridDim.x * groups_per_block;
    const int lid = threadIdx.x % kGroup;
    const int leader = lane - lid;
    // all groups of a warp run the same number of rounds (the shuffles need
    // every lane); a group past the last segment folds nothing
    const long long wbase = first - lane / kGroup;
    const long long count = wbase < p.nseg ? (p.nseg - wbase + step - 1) / step : 0;
#pragma unroll 1
    for (long long k0 = 0; k0 < count; k0 += kSegPipe) {
      // phase 1: the first round of every segment -- one vector, one head and
      // one tail element per lane -- with all kSegPipe segments' loads issued
      // before any is folded
      uint32_t r[kSegPipe][8];
      Elem hv[kSegPipe], tv[kSegPipe];
      bool hasv[kSegPipe], hash[kSegPipe], hast[kSegPipe], more = false;
      unsigned slot[kSegPipe];
#pragma unroll
      for (int j = 0; j < kSegPipe; ++j) {
        long long lo, hi;
        seg_bounds<T>(p, first + (k0 + j) * step, lo, hi);
        const SegGeo g = seg_geo<T>(p.in, lo, hi);
        hasv[j] = lid < g.nvec;
        hash[j] = lid < g.head;
        hast[j] = lid < g.tail;
        more |= g.nvec > kGroup || (kGroup < 8 && (g.head > kGroup || g.tail > kGroup));
        if (hasv[j]) ld_v8(g.body + (long long)lid * kVecBytes, r[j]);
        if (hash[j]) hv[j] = __ldg((const Elem*)g.p + lid);
        if (hast[j]) tv[j] = __ldg((const Elem*)(g.body + g.nvec * kVecBytes) + lid);
        // a long segment: the leader queues the rest of it (every lane of the
        // warp takes part in the broadcast)
        slot[j] = kNoSlot;
        if (p.use_q) {  // warp-uniform
          slot[j] = seg_reserve_warp(p, lid == 0 && g.nvec - kGroup > kLong, first + (k0 + j) * step,
                                     lo + g.head + (long long)kGroup * T::VE, lo + g.head + g.nvec * T::VE, T::VE,
                                     lane);
          if constexpr (kGroup > 1) slot[j] = __shfl_sync(0xffffffffu, slot[j], leader);
        }
      }
      Acc v[kSegPipe];
#pragma unroll
      for (int j = 0; j < kSegPipe; ++j) {
        Part<T> a[T::NA];
        init_parts<T>(a);
        uint32_t aux = 0;
        if (hasv[j]) fold_vec<T>(a, aux, r[j], 1);
        if (hash[j]) fold_elem<T>(a[0], aux, hv[j]);
        if (hast[j]) fold_elem<T>(a[T::NA - 1], aux, tv[j]);
        v[j] = thread_result<T>(a, aux);
      }
      // phase 2 (the rest of segments longer than one round that were not
      // queued; for groups narrower than 8 lanes also the head / tail elements
      // past the first): one code copy for all j, geometry recomputed
      if (more) {
#pragma unroll 1
        for (int j = 0; j < kSegPipe; ++j) {
          long long lo, hi;
          seg_bounds<T>(p, first + (k0 + j) * step, lo, hi);
          const SegGeo g = seg_geo<T>(p.in, lo, hi);
          unsigned sj = kNoSlot;
#pragma unroll
          for (int q = 0; q < kSegPipe; ++q)
            if (q == j) sj = slot[q];
          Part<T> a[T::NA];
          init_parts<T>(a);
          uint32_t aux = 0;
          bool any = false;
          if (g.nvec > kGroup && sj == kNoSlot) {
            fold_body<T, 4, kTail>(a, aux, g.body, lid + kGroup, g.nvec, kGroup);
            any = true;
          }
          if constexpr (kGroup < 8) {
            for (int h = lid + kGroup; h < g.head; h += kGroup) fold_elem<T>(a[0], aux, __ldg((const Elem*)g.p + h));
            for (int t = lid + kGroup; t < g.tail; t += kGroup)
              fold_elem<T>(a[T::NA - 1], aux, __ldg((const Elem*)(g.body + g.nvec * kVecBytes) + t));
            any |= g.head > kGroup || g.tail > kGroup;
          }
          if (any) {
            const Acc e = thread_result<T>(a, aux);
#pragma unroll
            for (int q = 0; q < kSegPipe; ++q)
              if (q == j) v[q] = T::comb(v[q], e);
          }
        }
      }
#pragma unroll
      for (int j = 0; j < kSegPipe; ++j) {
        const long long seg = first + (k0 + j) * step;
        Acc w = v[j];
        if constexpr (kGroup == 32) {
          w = T::warp(w);
        } else {
#pragma unroll
          for (int o = kGroup / 2; o > 0; o >>= 1) w = T::comb(w, shfl_xor(w, o));
        }
        if (lid == 0 && seg < p.nseg) {
          if (slot[j] != kNoSlot) ((Grid*)p.q.partials)[slot[j]] = T::to_grid(w);  // k_seg_finish writes out[seg]
          else seg_store<T>(p, seg, T::to_grid(w));
        }
      }
    }
  } else {
    __shared__ unsigned s_slot;
#pragma unroll 1
    for (long long seg = blockIdx.x; seg < p.nseg; seg += gridDim.x) {
      long long lo, hi;
      seg_bounds<T>(p, seg, lo, hi);
      const SegGeo g = seg_geo<T>(p.in, lo, hi);
      if (threadIdx.x == 0) {
        s_slot = kNoSlot;
        if (p.use_q && g.nvec - (long long)blockDim.x > kLong)
          s_slot = seg_reserve(p.q.hdr, p.q.items, p.q.longs, seg, lo + g.head + (long long)blockDim.x * T::VE,
                               lo + g.head + g.nvec * T::VE, T::VE);
      }
      __syncthreads();
      const unsigned sl = s_slot;
      Part<T> a[T::NA];
      init_parts<T>(a);
      uint32_t aux = 0;
      // a queued segment: only the first round here
      fold_body<T, 4, kTail>(a, aux, g.body, threadIdx.x, sl != kNoSlot ? (long long)blockDim.x : g.nvec, blockDim.x);
      if ((int)threadIdx.x < g.head) fold_elem<T>(a[0], aux, __ldg((const Elem*)g.p + threadIdx.x));
      if ((int)threadIdx.x < g.tail)
        fold_elem<T>(a[T::NA - 1], aux, __ldg((const Elem*)(g.body + g.nvec * kVecBytes) + threadIdx.x));
      const Grid gv = block_combine<T, BC_SHFL>(thread_result<T>(a, aux));
      if (threadIdx.x == 0) {
        if (sl != kNoSlot) ((Grid*)p.q.partials)[sl] = gv;
        else seg_store<T>(p, seg, gv);
      }
      __syncthreads();  // block_combine's shared scratch and s_slot are reused next iteration
    }
  }
  pdl_trigger();  // persistent grid: let the next kernel in only as this one finishes
}

// Queued chunks -> partials, one warp per chunk (persistent grid).
template <int DT, int OP>
__global__ void __launch_bounds__(256) k_seg_chunks(const SegParams p) {
  using T = Tr<DT, OP>;
  pdl_wait();
  unsigned n = *(volatile unsigned*)(p.q.hdr + 0);
  if (n > kSegQItems) n = kSegQItems;
  const int lane = threadIdx.x & 31;
  const unsigned warps = gridDim.x * (blockDim.x >> 5);
#pragma unroll 1
  for (unsigned i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n; i += warps) {
    const long long lo = p.q.items[2 * (size_t)i], hi = p.q.items[2 * (size_t)i + 1];
    if (hi <= lo) continue;  // a group partial's slot, or left empty (warp-uniform)
    Part<T> a[T::NA];
    init_parts<T>(a);
    uint32_t aux = 0;
    fold_range<T, 4>(a, aux, p.in, lo, hi, lane, 32);
    const typename T::Acc w = T::warp(thread_result<T>(a, aux));
    if (lane == 0) ((typename T::Grid*)p.q.partials)[i] = T::to_grid(w);
  }
  pdl_trigger();
}

// One warp per queued segment: its partials in order (the group's first round,
// then the chunks) -> out[seg]; the last block resets the queue for the next
// call on this stream.
template <int DT, int OP>
__global__ void __launch_bounds__(256) k_seg_finish(const SegParams p) {
  using T = Tr<DT, OP>;
  using Grid = typename T::Grid;
  pdl_wait();
  unsigned nl = *(volatile unsigned*)(p.q.hdr + 1);
  if (nl > kSegQLongs) nl = kSegQLongs;
  const int lane = threadIdx.x & 31;
  const unsigned warps = gridDim.x * (blockDim.x >> 5);
#pragma unroll 1
  for (unsigned j = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); j < nl; j += warps) {
    const long long seg = p.q.longs[3 * (size_t)j], base = p.q.longs[3 * (size_t)j + 1];
    const long long cnt = p.q.longs[3 * (size_t)j + 2];
    Grid x = T::gident();
    for (long long i = lane; i < cnt; i += 32) x = T::gcomb(x, __ldcg((const Grid*)p.q.partials + base + i));
    x = T::gwarp(x);
    if (lane == 0) seg_store<T>(p, seg, x);
  }
  __syncthreads();
  if (threadIdx.x == 0 && ticket_acq_rel(p.q.hdr + 2) == gridDim.x - 1) {
    p.q.hdr[0] = 0u;
    p.q.hdr[1] = 0u;
    p.q.hdr[2] = 0u;
  }
  pdl_trigger();
}

// Uniform rows of nv 32-byte vectors that all start on 32-byte boundaries
// (row bytes a multiple of 32, aligned input) and are at most 256 bytes: one
// thread per row issues every load of its row at once (the group kernels'
// first round plus a dependent second round cost a load latency per row),
// folds them with the vector tree and writes out[row].  Rows of NV = 1, 2 or 4
// vectors take R = 8 / NV rows per thread per step (rows r, r + stride, ...),
// so eight 32-byte loads are in flight per thread whatever the row length.
// One-wave grid striding over the rows.  NV = 0: the row length is a runtime
// value (<= 8 vectors), one row per step.
#ifndef RB_ROWS_BLOCK
#define RB_ROWS_BLOCK 128
#endif
template <int DT, int OP, int NV>
__global__ void __launch_bounds__(RB_ROWS_BLOCK) k_rows_aligned(const SegParams p) {
  using T = Tr<DT, OP>;
  constexpr int R = NV > 0 ? 8 / NV : 1;
  pdl_wait();
  const int nv = NV > 0 ? NV : p.rows_nv;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long row_bytes = (long long)nv * kVecBytes;
#pragma unroll 1
  for (long long row0 = (long long)blockIdx.x * blockDim.x + threadIdx.x; row0 < p.nseg; row0 += stride * R) {
    uint32_t r[8][8];
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const long long row = row0 + j * stride;
      const char* rp = p.in + row * row_bytes;
#pragma unroll
      for (int v = 0; v < (NV > 0 ? NV : 8); ++v)
        if (row < p.nseg && v < nv) ld_v8(rp + v * kVecBytes, r[j * (NV > 0 ? NV : 0) + v]);
    }
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const long long row = row0 + j * stride;
      if (row >= p.nseg) break;
      Part<T> a[T::NA];
      init_parts<T>(a);
      uint32_t aux = 0;
#pragma unroll
      for (int v = 0; v < (NV > 0 ? NV : 8); ++v)
        if (v < nv) fold_vec<T>(a, aux, r[j * (NV > 0 ? NV : 0) + v], v);
      seg_store<T>(p, row, T::to_grid(thread_result<T>(a, aux)));
    }
  }
  pdl_trigger();
}

template <int DT, int OP, int NV>
cudaError_t launch_rows_aligned(const SegParams& p, int sms, cudaStream_t s) {
  const int per_sm = blocks_per_sm((const void*)k_rows_aligned<DT, OP, NV>, RB_ROWS_BLOCK, 0);
  long long grid = (p.nseg + RB_ROWS_BLOCK - 1) / RB_ROWS_BLOCK;
  if (grid > (long long)sms * per_sm) grid = (long long)sms * per_sm;
  return seg_launch(k_rows_aligned<DT, OP, NV>, grid < 1 ? 1 : grid, RB_ROWS_BLOCK, p, s);
}

// Uniform rows of 1, 2, 4, 8, 16 or 32 KB (L = 32 << LV vectors) on 32-byte
// boundaries: the flat kernel's tile walk over the batch.  Block b reads the
// contiguous 32 KB tile b exactly as k_reduce does (256 threads x 4 loads of
// 256 bits, all in flight); each warp-load of 32 vectors lies inside one row,
// so every (load, warp) pair is warp-reduced on its own, the tile's 32
// warp-vector partials meet in shared memory, and warp 0 combines each row's
// WPR = L / 32 consecutive partials with a butterfly of width WPR (fixed tree,
// deterministic, no atomics).  The tile holds 32 / WPR whole rows.  LV < 0:
// rows of 1-16 vectors (32-512 bytes), 32 / L rows per warp-load, each reduced
// by a butterfly of width L and stored by its first lane (no shared memory).
template <int DT, int OP, int LV>
__global__ void __launch_bounds__(256) k_rows_tiled(const SegParams p) {
  using T = Tr<DT, OP>;
  using Acc = typename T::Acc;
  constexpr int U = 4, B = 256, WPR = LV >= 0 ? 1 << LV : 1;
  constexpr long long kTile = (long long)U * B;  // vectors
  __shared__ Acc part[U * (B / 32)];
  pdl_wait();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const long long total = p.nseg << (5 + LV);  // vectors in the batch
#pragma unroll 1
  for (long long tile = blockIdx.x; tile * kTile < total; tile += gridDim.x) {
    const long long left = total - tile * kTile;  // a multiple of the row length
    const char* base = p.in + (tile * kTile + threadIdx.x) * kVecBytes;
    uint32_t r[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u)
      if ((long long)(u * B + threadIdx.x) < left) ld_v8(base + (size_t)u * B * kVecBytes, r[u]);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      Part<T> a[T::NA];
      init_parts<T>(a);
      uint32_t aux = 0;
      const bool valid = (long long)(u * B + threadIdx.x) < left;
      if (valid) fold_vec<T>(a, aux, r[u], 0);
      if constexpr (LV < 0) {
        // rows of 1-16 vectors: 32 / L rows per warp-load, a butterfly of width L
        Acc w = thread_result<T>(a, aux);
#pragma unroll
        for (int o = (1 << (LV + 5)) / 2; o > 0; o >>= 1) w = T::comb(w, shfl_xor(w, o));
        if (valid && (lane & ((1 << (LV + 5)) - 1)) == 0)
          seg_store<T>(p, (tile * kTile + u * B + threadIdx.x) >> (LV + 5), T::to_grid(w));
      } else {
        const Acc w = T::warp(thread_result<T>(a, aux));
        if (lane == 0) part[u * (B / 32) + wid] = w;
      }
    }
    if constexpr (LV >= 0) {
      __syncthreads();
      if (wid == 0) {
        Acc x = part[lane];
#pragma unroll
        for (int o = WPR / 2; o > 0; o >>= 1) x = T::comb(x, shfl_xor(x, o));
        const long long row = (tile << (5 - LV)) + (lane >> LV);
        if ((lane & (WPR - 1)) == 0 && row < p.nseg) seg_store<T>(p, row, T::to_grid(x));
      }
      __syncthreads();  // part[] is reused by the next tile
    }
  }
  pdl_trigger();
}

// Uniform rows of a whole number (>= 2) of 32 KB tiles, 32-byte aligned, and
// enough rows to fill the GPU (host side): one block per row walks the row's
// tiles with k_reduce's access pattern (4 loads of 256 bits per thread in
// flight), then the "Vs" block combine.  Rows beyond the grid are strided.
template <int DT, int OP>
__global__ void __launch_bounds__(256) k_rows_tiled_big(const SegParams p) {
  using T = Tr<DT, OP>;
  constexpr int U = 4, B = 256;
  constexpr long long kTile = (long long)U * B;  // vectors
  pdl_wait();
  const long long row_vecs = (long long)p.rows_tiled_vecs;
#pragma unroll 1
  for (long long row = blockIdx.x; row < p.nseg; row += gridDim.x) {
    Part<T> a[T::NA];
    init_parts<T>(a);
    uint32_t aux = 0;
    const char* base = p.in + (row * row_vecs + threadIdx.x) * kVecBytes;
#pragma unroll 1
    for (long long v = 0; v < row_vecs; v += kTile) {
      uint32_t r[U][8];
#pragma unroll
      for (int u = 0; u < U; ++u) ld_v8(base + (v + (long long)u * B) * kVecBytes, r[u]);
#pragma unroll
      for (int u = 0; u < U; ++u) fold_vec<T>(a, aux, r[u], u);
    }
    const typename T::Grid g = block_combine<T, BC_SHFL>(thread_result<T>(a, aux));
    if (threadIdx.x == 0) seg_store<T>(p, row, g);
    __syncthreads();  // block_combine's shared scratch is reused by the next row
  }
  pdl_trigger();
}

template <int DT, int OP, int LV>
cudaError_t launch_rows_tiled_lv(const SegParams& p, cudaStream_t s) {
  const long long tiles = ((p.nseg << (5 + LV)) + 1023) >> 10;  // one block per 32 KB tile
  const long long grid = tiles < (1ll << 30) ? tiles : (1ll << 30);
  return seg_launch(k_rows_tiled<DT, OP, LV>, grid < 1 ? 1 : grid, 256, p, s);
}

template <int DT, int OP>
cudaError_t launch_rows_tiled(const SegParams& p, cudaStream_t s) {
  if (p.rows_tiled_vecs > 0) {
    const long long grid = p.nseg < (1ll << 30) ? p.nseg : (1ll << 30);
    return seg_launch(k_rows_tiled_big<DT, OP>, grid, 256, p, s);
  }
  switch (p.rows_tiled - 6) {  // LV = log2(row vectors) - 5
    case -5: return launch_rows_tiled_lv<DT, OP, -5>(p, s);
    case -4: return launch_rows_tiled_lv<DT, OP, -4>(p, s);
    case -3: return launch_rows_tiled_lv<DT, OP, -3>(p, s);
    case -2: return launch_rows_tiled_lv<DT, OP, -2>(p, s);
    case -1: return launch_rows_tiled_lv<DT, OP, -1>(p, s);
    case 0: return launch_rows_tiled_lv<DT, OP, 0>(p, s);
    case 1: return launch_rows_tiled_lv<DT, OP, 1>(p, s);
    case 2: return launch_rows_tiled_lv<DT, OP, 2>(p, s);
    case 3: return launch_rows_tiled_lv<DT, OP, 3>(p, s);
    case 4: return launch_rows_tiled_lv<DT, OP, 4>(p, s);
    case 5: return launch_rows_tiled_lv<DT, OP, 5>(p, s);
  }
  return cudaErrorInvalidValue;
}

template <class K>
cudaError_t seg_launch(K kernel, long long grid, int block, const SegParams& p, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kernel, p);
}

template <int DT, int OP, int kGroup, bool kTail>
cudaError_t launch_segmented_group(const SegParams& p, int block, int sms, cudaStream_t s) {
  const int per_sm = blocks_per_sm((const void*)k_segmented<DT, OP, kGroup, kTail>, block, 0);
  const long long per_block = kGroup > 0 ? block / kGroup : 1;
  long long grid = (p.nseg + per_block - 1) / per_block;
  const long long cap = (long long)sms * per_sm;  // one full wave
  if (grid > cap) grid = cap;
  if (grid < 1) grid = 1;
  return seg_launch(k_segmented<DT, OP, kGroup, kTail>, grid, block, p, s);
}

template <int DT, int OP, bool kTail>
cudaError_t launch_segmented_groups(const SegParams& p, int group, int block, int sms, cudaStream_t s) {
  if (group == 1) return launch_segmented_group<DT, OP, 1, kTail>(p, block, sms, s);
  if (group == 8) return launch_segmented_group<DT, OP, 8, kTail>(p, block, sms, s);
  if (group == 32) return launch_segmented_group<DT, OP, 32, kTail>(p, block, sms, s);
  return launch_segmented_group<DT, OP, 0, kTail>(p, block, sms, s);
}

template <int DT, int OP>
cudaError_t launch_segmented_op(const SegParams& p, int group, int block, cudaStream_t s) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (p.rows_tiled > 0) return launch_rows_tiled<DT, OP>(p, s);
  if (p.rows_nv > 0) {
    if constexpr (OP != OP_SUMACC) {  // several rows per thread: the accurate pairs would not fit
      if (p.rows_nv == 1) return launch_rows_aligned<DT, OP, 1>(p, sms, s);
      if (p.rows_nv == 2) return launch_rows_aligned<DT, OP, 2>(p, sms, s);
      if (p.rows_nv == 4) return launch_rows_aligned<DT, OP, 4>(p, sms, s);
    }
    return launch_rows_aligned<DT, OP, 0>(p, sms, s);
  }
  cudaError_t e = p.tail ? launch_segmented_groups<DT, OP, true>(p, group, block, sms, s)
                         : launch_segmented_groups<DT, OP, false>(p, group, block, sms, s);
  if (e != cudaSuccess || !p.use_q) return e;
  const int chunk_per_sm = blocks_per_sm((const void*)k_seg_chunks<DT, OP>, 256, 0);
  e = seg_launch(k_seg_chunks<DT, OP>, (long long)sms * chunk_per_sm, 256, p, s);
  if (e != cudaSuccess) return e;
  return seg_launch(k_seg_finish<DT, OP>, sms, 256, p, s);
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
