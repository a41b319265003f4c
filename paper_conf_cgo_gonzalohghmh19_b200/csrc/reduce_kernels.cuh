// reduce_kernels.cuh -- the reduction kernels (steps S2-S6 of DESIGN.md) as
// templates, instantiated per dtype in reduce_{i32,f32,f64}.cu.
//
// k_reduce<DT, OP, U, BC>: one kernel covers the paper's warp-only, single-block
// and grid-level versions (Fig. 6):
//   * partition (S2): the 32-byte-aligned body is cut into tiles of
//     blockDim.x * U vectors; tiles go to blocks ("Global Atomic Tile
//     Distribute", DT at grid level) and, inside a tile, vectors go to threads
//     with stride blockDim.x ("Stride Distribute", DS at thread level) -- the
//     large-array winners (b), (e) of P:L687 -- so each warp load instruction
//     covers 1 KB contiguous.  Each thread issues its U 256-bit loads before
//     consuming any (memory-level parallelism), folding into NA independent
//     register accumulators (Fig. 1(a)'s `accum += in[i]`).
//     With grid == tiles (the default) every block does exactly one tile and
//     the hardware block scheduler balances the tail across the 148 SMs; with
//     a smaller grid, blocks loop over tiles (persistent, Catanzaro-style
//     two-stage); grid == 1 is the single-block / warp-only path.
//   * head (< 32 B before the aligned body) and tail (< 32 B after it) are
//     folded by the last block's threads 0..7 and 8..15.
//   * warp / block combine (S3, S4): block_combine<BC>.
//   * grid combine (S5) and finalise (S6): by desc.gc, see grid_combine().
#pragma once
#include <cooperative_groups.h>
#include <map>
#include <mutex>
#include <tuple>
#include <type_traits>
#include "reduce_device.cuh"
#include "reduce_internal.h"

namespace rb {

struct KParams {
  const char* in;
  const char* body;
  unsigned long long body_vecs;
  long long tiles;
  int head, tail;
  void* out;
  int raw_out;
  int gc;
  void* slots;
  int nslots;
  unsigned* ticket;
  void* partials;
  TeamArgs team;
  int early;
  int pf_stride;   // early != 0: blocks below pf_stride prefetch tiles blockIdx + k*pf_stride,
  int pf_tiles;    //   k < pf_tiles, into L2 before the wait (set by launch_kernel)
  unsigned trig_window;  // blocks of the last ~wave (kPdlBlocksPerSm x SMs), set by launch_kernel
};

// Polling loops spin without sleeping for this many cycles (~10 us), then
// back off with nanosleep: a sleep per miss added 0.3-1 us per call to the
// FLAGS combine (profiles/r02_flags_ab.jsonl); long waits still yield.
constexpr long long kSpinCycles = 20000;

// ---- one-shot cross-GPU combine through peer memory ------
// Executed by ONE thread of the block that owns this rank's raw result x.
// Flag-in-data protocol (as NCCL's "LL"): every 4-byte word of x travels with
// the call's epoch in the same aligned 8-byte pair {word, epoch}, written to
// slot [parity][rank] of every member's buffer (P2P stores over NVLink).  A
// reader polls its own buffer until every pair of every slot 0..k-1 carries
// the epoch, then combines the k values in rank order (deterministic for a
// fixed team).  No fences: an 8-byte pair is written and read as one access,
// so a matching epoch implies the word beside it.  Measured on B200 (tools/
// probes/probe_fence.cu): fence.acq_rel.sys ~1.1 us each; the release/acquire
// version of this exchange cost ~5 us per call, this one ~1 us.
// Parity double-buffering: a rank can reuse parity p only after every member
// has written its pairs for the following call, i.e. after everyone finished
// reading parity p.
__device__ __forceinline__ void st_pairs_sys(unsigned* p, unsigned a, unsigned b, unsigned e) {
  asm volatile("st.relaxed.sys.global.v4.u32 [%0], {%1, %2, %3, %4};" :: "l"(p), "r"(a), "r"(e), "r"(b), "r"(e)
               : "memory");
}
__device__ __forceinline__ void ld_pairs_sys(const unsigned* p, unsigned& a, unsigned& fa, unsigned& b, unsigned& fb) {
  asm volatile("ld.relaxed.sys.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(a), "=r"(fa), "=r"(b), "=r"(fb) : "l"(p)
               : "memory");
}

// Scalars by value (taking the address of a kernel-parameter struct would copy
// it to the stack in every thread of every block -- measured: -18 % bandwidth).
template <class T>
__device__ __noinline__ typename T::Grid team_exchange(typename T::Grid x, char* const* bufs, int k, int rank) {
  using Grid = typename T::Grid;
  static_assert(sizeof(Grid) <= 16 && sizeof(Grid) % 4 == 0, "team slot holds <= 4 words");
  constexpr int NW = sizeof(Grid) / 4;  // data words
  constexpr int NV = (NW + 1) / 2;      // 16-byte stores of {w, e, w, e}
  // advance this rank's call counter (every member calls in the same order, so
  // the counters agree); 0 means "never written" and is skipped so that the
  // parity still alternates across the wrap: ..., 2^32-1 (odd), 2 (even), 3, ...
  volatile unsigned* ctr = (volatile unsigned*)(bufs[rank] + kTeamEpochOff);
  unsigned epoch = *ctr + 1;
  if (epoch == 0) epoch = 2;
  *ctr = epoch;
  const int par = epoch & 1;
  unsigned w[4] = {0u, 0u, 0u, 0u};
  memcpy(w, &x, sizeof(Grid));
  for (int j = 0; j < k; ++j) {
    if (j == rank) continue;  // the own value never leaves the register
    unsigned* dst = (unsigned*)(bufs[j] + ((size_t)par * kTeamMaxRanks + rank) * kTeamSlotBytes);
#pragma unroll
    for (int v = 0; v < NV; ++v) st_pairs_sys(dst + 4 * v, w[2 * v], w[2 * v + 1], epoch);
  }
  const char* own = bufs[rank];
  Grid acc = T::gident();
  for (int j = 0; j < k; ++j) {
    if (j == rank) {
      acc = T::gcomb(acc, x);
      continue;
    }
    const unsigned* src = (const unsigned*)(own + ((size_t)par * kTeamMaxRanks + j) * kTeamSlotBytes);
    unsigned r[4] = {0u, 0u, 0u, 0u};
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      unsigned fa, fb;
      ld_pairs_sys(src + 4 * v, r[2 * v], fa, r[2 * v + 1], fb);
      if (fa != epoch || fb != epoch) {
        const long long t0 = clock64();
        do {
          if (clock64() - t0 > kSpinCycles) __nanosleep(64);  // spin first: a sleep costs ~0.5 us of latency
          // a member that never arrives must not hang the GPU: after ~2^35
          // cycles (> 15 s) abort the kernel -- the error surfaces at the sync
          if (clock64() - t0 > (1ll << 35)) __trap();
          ld_pairs_sys(src + 4 * v, r[2 * v], fa, r[2 * v + 1], fb);
        } while (fa != epoch || fb != epoch);
      }
    }
    Grid y;
    memcpy(&y, r, sizeof(Grid));
    acc = T::gcomb(acc, y);
  }
  return acc;
}

// ---- cross-GPU combine through NVLink SHARP multicast -----
// One thread of the block that owns this rank's raw result x.  bufs[j]: rank
// j's copy of the NCCL symmetric window (unicast); mc: the window's multicast
// address -- a store or reduction there reaches every rank's copy through the
// NVSwitch, a multimem.ld_reduce returns the reduction of all copies.
//  mode 1: x goes to the own copy's slot [parity]; one multimem.red.release
//          adds 1 to every copy's barrier counter (the release orders the slot
//          store before it); when the own counter reaches calls * k every rank
//          has published, and ONE multimem.ld_reduce reduces the k slots in the
//          switch.  double-double values (no switch op) are read from the k
//          copies in rank order instead.
//  mode 2: one multimem.st puts {word, epoch} pairs into slot [parity][rank]
//          of every copy (flag-in-data, no fence, as team_exchange); the own
//          copy is polled until all k slots carry the epoch and combined in
//          rank order: deterministic for a fixed team.
// Parity double-buffering as in team_exchange: a slot is rewritten two calls
// later, after every rank passed the intervening call.
template <class T>
__device__ __forceinline__ bool mc_ld_reduce(const char* a, typename T::Grid& r) {
  using G = typename T::Grid;
  if constexpr (std::is_same<G, double>::value) {
    double v;
    asm volatile("multimem.ld_reduce.relaxed.sys.global.add.f64 %0, [%1];" : "=d"(v) : "l"(a) : "memory");
    r = v;
    return true;
  } else if constexpr (std::is_same<G, uint32_t>::value) {
    uint32_t v;
    if constexpr (T::kOp == OP_SUM)
      asm volatile("multimem.ld_reduce.relaxed.sys.global.add.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
    else if constexpr (T::kOp == OP_MIN)
      asm volatile("multimem.ld_reduce.relaxed.sys.global.min.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
    else
      asm volatile("multimem.ld_reduce.relaxed.sys.global.max.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
    r = v;
    return true;
  } else if constexpr (std::is_same<G, int32_t>::value) {
    int32_t v;
    if constexpr (T::kOp == OP_MIN)
      asm volatile("multimem.ld_reduce.relaxed.sys.global.min.s32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
    else
      asm volatile("multimem.ld_reduce.relaxed.sys.global.max.s32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
    r = v;
    return true;
  } else if constexpr (std::is_same<G, unsigned long long>::value) {
    unsigned long long v;
    if constexpr (T::kOp == OP_MIN)
      asm volatile("multimem.ld_reduce.relaxed.sys.global.min.u64 %0, [%1];" : "=l"(v) : "l"(a) : "memory");
    else
      asm volatile("multimem.ld_reduce.relaxed.sys.global.max.u64 %0, [%1];" : "=l"(v) : "l"(a) : "memory");
    r = v;
    return true;
  } else {
    return false;
  }
}

template <class T>
__device__ __noinline__ typename T::Grid nvls_exchange(typename T::Grid x, char* const* bufs, int k, int rank, int mode) {
  using Grid = typename T::Grid;
  static_assert(sizeof(Grid) <= 16 && sizeof(Grid) % 4 == 0, "nvls slot holds <= 4 words");
  constexpr int NW = sizeof(Grid) / 4;
  constexpr int NV = (NW + 1) / 2;
  char* const mc = bufs[k];
  volatile unsigned* c = (volatile unsigned*)bufs[k + 1];
  char* own = bufs[rank];
  unsigned w[4] = {0u, 0u, 0u, 0u};
  memcpy(w, &x, sizeof(Grid));
  if (mode == 1) {
    const unsigned calls = c[1] + 1;
    c[1] = calls;
    const size_t slot = kNvlsRedOff + (size_t)(calls & 1) * 16;
    asm volatile("st.relaxed.sys.global.v4.u32 [%0], {%1, %2, %3, %4};" :: "l"(own + slot), "r"(w[0]), "r"(w[1]),
                 "r"(w[2]), "r"(w[3]) : "memory");
    asm volatile("multimem.red.release.sys.global.add.u32 [%0], 1;" :: "l"(mc + kNvlsCtrOff) : "memory");
    const unsigned target = calls * (unsigned)k;
    unsigned got;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(got) : "l"(own + kNvlsCtrOff) : "memory");
    if ((int)(got - target) < 0) {
      const long long t0 = clock64();
      do {
        if (clock64() - t0 > kSpinCycles) __nanosleep(64);  // spin first: a sleep costs ~0.5 us of latency
        if (clock64() - t0 > (1ll << 35)) __trap();  // a member that never arrives: abort, not hang
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(got) : "l"(own + kNvlsCtrOff) : "memory");
      } while ((int)(got - target) < 0);
    }
    Grid r;
    if (mc_ld_reduce<T>(mc + slot, r)) return r;
    Grid acc = T::gident();
    for (int j = 0; j < k; ++j) {
      unsigned v[4];
      asm volatile("ld.relaxed.sys.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
                   : "l"(bufs[j] + slot) : "memory");
      Grid y;
      memcpy(&y, v, sizeof(Grid));
      acc = T::gcomb(acc, y);
    }
    return acc;
  }
  // mode 2: multicast flag-in-data
  unsigned epoch = c[0] + 1;
  if (epoch == 0) epoch = 2;  // 0 means "never written"; keep the parity alternating across the wrap
  c[0] = epoch;
  const int par = epoch & 1;
  char* dst = mc + kNvlsLLOff + ((size_t)par * kTeamMaxRanks + rank) * kTeamSlotBytes;
#pragma unroll
  for (int v = 0; v < NV; ++v)
    asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1, %2, %3, %4};" :: "l"(dst + 16 * v),
                 "f"(__uint_as_float(w[2 * v])), "f"(__uint_as_float(epoch)), "f"(__uint_as_float(w[2 * v + 1])),
                 "f"(__uint_as_float(epoch)) : "memory");
  Grid acc = T::gident();
  for (int j = 0; j < k; ++j) {
    if (j == rank) {
      acc = T::gcomb(acc, x);
      continue;
    }
    const unsigned* src = (const unsigned*)(own + kNvlsLLOff + ((size_t)par * kTeamMaxRanks + j) * kTeamSlotBytes);
    unsigned r[4] = {0u, 0u, 0u, 0u};
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      unsigned fa, fb;
      ld_pairs_sys(src + 4 * v, r[2 * v], fa, r[2 * v + 1], fb);
      if (fa != epoch || fb != epoch) {
        const long long t0 = clock64();
        do {
          if (clock64() - t0 > kSpinCycles) __nanosleep(64);  // spin first: a sleep costs ~0.5 us of latency
          if (clock64() - t0 > (1ll << 35)) __trap();
          ld_pairs_sys(src + 4 * v, r[2 * v], fa, r[2 * v + 1], fb);
        } while (fa != epoch || fb != epoch);
      }
    }
    Grid y;
    memcpy(&y, r, sizeof(Grid));
    acc = T::gcomb(acc, y);
  }
  return acc;
}

// The cross-rank step: scalars by value into the __noinline__ exchanges (a
// reference to the parameter struct would copy it to the stack).
#define RB_CROSS_RANK(T, g, t)                                                              \
  ((t).nvls ? nvls_exchange<T>((g), (t).bufs, (t).k, (t).rank, (t).nvls)                     \
            : team_exchange<T>((g), (t).bufs, (t).k, (t).rank))

template <class T>
__device__ __forceinline__ void store_out(typename T::Grid g, const KParams& p) {
  if (p.team.k > 0) g = RB_CROSS_RANK(T, g, p.team);
  if (p.raw_out) *(typename T::Grid*)p.out = g;
  else T::finalize(g, p.out);
}

// GC_FLAGS: flag-in-data partial records polled by one fixed block -- no
// atomic, no fence, no ticket.  Every block but the last stores its partial as
// {word, epoch} pairs (one 16-byte relaxed store per two words: each aligned
// 8-byte pair is written and read as one access, so a matching epoch implies
// the word beside it -- the protocol of team_exchange, inside one GPU).  Block
// G-1 (dispatched last, so it rarely waits) polls records 0..G-2 with loads in
// flight, combines them in index order with its own value last and a fixed
// tree (deterministic for a fixed launch shape), writes the result and
// publishes the next epoch.  The epoch word (p.ticket) is read by every block
// after the dependency resolves and advanced only by the poller, after every
// record of the call was consumed; a record from an older call carries an
// older epoch.  When the 32-bit epoch would wrap, the poller zeroes the whole
// record area (its size in bytes is the 64-bit word at p.ticket + 2) first.
// Replaces the ATOMIC chain red -> release -> ticket -> exchange (three L2
// round trips after the loads) by one store and one poll (B200 probe,
// tools/probes/probe_mid.cu "flags_fixed": -1.0 to -2.1 us per call at 1-64 MB).
// (Scalars by value, as the exchanges below: a reference to the kernel's
// parameter struct in a non-inlined function would copy it to the stack.)
template <class T>
__device__ __noinline__ void flags_combine(typename T::Grid g, unsigned ep, char* const rec, unsigned* const ticket,
                                           void* const out, const int raw_out, const TeamArgs team) {
  using Grid = typename T::Grid;
  static_assert(sizeof(Grid) <= 16 && sizeof(Grid) % 4 == 0, "a record holds <= 4 words");
  constexpr int NW = sizeof(Grid) / 4;
  constexpr int NV = (NW + 1) / 2;  // 16-byte stores {w, e, w, e} per record
#ifndef RB_FLAGS_KB
#define RB_FLAGS_KB 4
#endif
#ifndef RB_FLAGS_SLEEP
#define RB_FLAGS_SLEEP 64
#endif
  constexpr int KB = NV == 1 ? RB_FLAGS_KB : 2;  // records in flight per thread
  const unsigned G1 = gridDim.x - 1;
  if (blockIdx.x != G1) {
    if (threadIdx.x == 0) {
      unsigned w[4] = {0u, 0u, 0u, 0u};
      memcpy(w, &g, sizeof(Grid));
#pragma unroll
      for (int v = 0; v < NV; ++v) st_pairs_gpu(rec + ((size_t)blockIdx.x * NV + v) * 16, w[2 * v], w[2 * v + 1], ep);
    }
    return;
  }
  __shared__ unsigned s_ep;
  __shared__ Grid s_own;
  __shared__ Grid gpart[32];
  if (threadIdx.x == 0) {
    s_ep = ep;
    s_own = g;
  }
  __syncthreads();
  const unsigned e = s_ep;
  const unsigned B = blockDim.x;
  Grid x = T::gident();
#pragma unroll 1
  for (unsigned i0 = threadIdx.x; i0 < G1; i0 += KB * B) {
    uint4 r[KB][NV];
#pragma unroll
    for (int j = 0; j < KB; ++j)
      if (i0 + j * B < G1)
#pragma unroll
        for (int v = 0; v < NV; ++v) r[j][v] = ld_pairs_gpu(rec + ((size_t)(i0 + j * B) * NV + v) * 16);
#pragma unroll
    for (int j = 0; j < KB; ++j) {
      if (i0 + j * B < G1) {
        unsigned w[4] = {0u, 0u, 0u, 0u};
#pragma unroll
        for (int v = 0; v < NV; ++v) {
          if (r[j][v].y != e || r[j][v].w != e) {
            const long long t0 = clock64();
            do {
              if (RB_FLAGS_SLEEP > 0 && clock64() - t0 > kSpinCycles) __nanosleep(RB_FLAGS_SLEEP);
              // a block that never publishes (a bug, not a race) must not hang the GPU
              if (clock64() - t0 > (1ll << 35)) __trap();
              r[j][v] = ld_pairs_gpu(rec + ((size_t)(i0 + j * B) * NV + v) * 16);
            } while (r[j][v].y != e || r[j][v].w != e);
          }
          w[2 * v] = r[j][v].x;
          w[2 * v + 1] = r[j][v].z;
        }
        Grid y;
        memcpy(&y, w, sizeof(Grid));
        x = T::gcomb(x, y);
      }
    }
  }
  if (threadIdx.x == G1 % B) x = T::gcomb(x, s_own);  // index G1 comes last in its thread's sequence
  x = T::gwarp(x);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (B + 31) >> 5;
  if (lane == 0) gpart[wid] = x;
  __syncthreads();
  if (wid == 0) {
    Grid y = lane < nw ? gpart[lane] : T::gident();
    y = T::gwarp(y);
    if (lane == 0) {
      if (team.k > 0) y = RB_CROSS_RANK(T, y, team);
      if (raw_out) *(Grid*)out = y;
      else T::finalize(y, out);
    }
  }
  if (e != 0xFFFFFFFFu) {
    if (threadIdx.x == 0) st_relaxed_u32(ticket, e);
    return;
  }
  // epoch wrap: no record may keep a value that a later epoch could match
  const unsigned long long cap = *(const unsigned long long*)(ticket + 2);
#pragma unroll 1
  for (unsigned long long o = (unsigned long long)threadIdx.x * 16; o + 16 <= cap; o += (unsigned long long)B * 16)
    *(uint4*)(rec + o) = make_uint4(0u, 0u, 0u, 0u);
  __syncthreads();
  if (threadIdx.x == 0) st_relaxed_u32(ticket, 0u);
}

template <class T>
__device__ __forceinline__ void grid_combine(typename T::Grid g, const KParams& p, unsigned ep) {
  using Grid = typename T::Grid;
  __shared__ int s_last;
  if (p.gc == GC_FLAGS) {
    flags_combine<T>(g, ep, (char*)p.partials, p.ticket, p.out, p.raw_out, p.team);
    return;
  }
  if (p.gc == GC_DIRECT) {
    if (threadIdx.x == 0) store_out<T>(g, p);
    return;
  }
  if (p.gc == GC_CLUSTER) {
    // CTA partials meet in CTA 0's shared memory over DSMEM.  The first
    // cluster-barrier phase (arrived at kernel start, see k_reduce) guarantees
    // CTA 0 has started before anyone writes into its shared memory; the
    // second (release/acquire) orders the remote stores before CTA 0 reads.
    namespace cg = cooperative_groups;
    __shared__ Grid cl_vals[16];
    cg::cluster_group cluster = cg::this_cluster();
    const unsigned r = cluster.block_rank();
    cluster_wait();
    if (threadIdx.x == 0) cluster.map_shared_rank(&cl_vals[0], 0)[r] = g;
    cluster.sync();
    if (r == 0 && threadIdx.x < 32) {
      const unsigned C = cluster.num_blocks();
      Grid x = threadIdx.x < C ? cl_vals[threadIdx.x] : T::gident();
      x = T::gwarp(x);
      if (threadIdx.x == 0) store_out<T>(x, p);
    }
    return;
  }
  if (p.gc == GC_TWO_PASS) {  // Listing 1: Return[blockIdx.x] = ...; second launch reduces
    if (threadIdx.x == 0) ((Grid*)p.partials)[blockIdx.x] = g;
    return;
  }
  if constexpr (HasPackedTicket<T>::value) {
    // int32 sums: Listing 2's `atomicAdd(Return, ...)` and the ticket
    // in one 64-bit atomic add on slot 0: bits 48-63 count the blocks, bits
    // 0-31 hold the sum mod 2^32 and bits 32-47 absorb its carries (at most one
    // per block, so < 2^16 for grids below 2^16).  The block that sees count
    // G-1 owns the complete sum in old + add -- no release fence before a
    // separate ticket, no second round trip to collect slots (B200 probe,
    // tools/probes/probe_mid.cu: -0.9 to -1.5 us per call at 1-64 MB).  It
    // resets the word for the next call.
    if (p.gc == GC_ATOMIC && gridDim.x < 65536u) {
      if (threadIdx.x == 0) {
        const unsigned long long add = (1ull << 48) | (unsigned long long)(uint32_t)g;
        const unsigned long long old = atomicAdd((unsigned long long*)p.slots, add);
        if ((unsigned)(old >> 48) == gridDim.x - 1) {
          atomicExch((unsigned long long*)p.slots, 0ull);
          store_out<T>((Grid)(uint32_t)(old + add), p);
        }
      }
      return;
    }
  }
  if (p.gc == GC_ATOMIC) {
    // Listing 2's `atomicAdd(Return, ...)` per block, spread over
    // nslots accumulators on separate L2 lines; the ticket's last holder
    // collects the slots (atomicExch resets them to the identity, so no memset
    // is ever needed) and publishes the result.
    if (threadIdx.x == 0) {
      Grid* slot = (Grid*)((char*)p.slots + (size_t)(blockIdx.x & (p.nslots - 1)) * kSlotBytes);  // nslots: power of 2
      T::gred(slot, g);
      const unsigned tk = ticket_acq_rel(p.ticket);  // release: the red above; acquire: everyone's
      s_last = (tk == gridDim.x - 1);
    }
    __syncthreads();
    if (s_last && threadIdx.x < 32) {
      const int lane = threadIdx.x;
      Grid x = T::gident();
      if (lane < p.nslots) x = T::gexch((Grid*)((char*)p.slots + (size_t)lane * kSlotBytes), T::gident());
      x = T::gwarp(x);
      if (lane == 0) {
        store_out<T>(x, p);
        atomicExch(p.ticket, 0u);
      }
    }
    return;
  }
  // GC_LAST_BLOCK: partials + ticket; the last block reduces them in a fixed
  // order (deterministic; the only atomic touches the integer ticket).
  if (threadIdx.x == 0) {
    ((Grid*)p.partials)[blockIdx.x] = g;
    const unsigned tk = ticket_acq_rel(p.ticket);  // release: the store above; acquire: everyone's
    s_last = (tk == gridDim.x - 1);
  }
  __syncthreads();
  if (s_last) {
    Grid x = reduce_grid_values<T>((const Grid*)p.partials, gridDim.x);
    if (threadIdx.x == 0) {
      store_out<T>(x, p);
      atomicExch(p.ticket, 0u);
    }
  }
}

template <int DT, int OP, int U, int BC, int STAGE>
__global__ void __launch_bounds__(max_block_threads(DT, OP, U, STAGE),
                                  min_blocks_hint(DT, OP, U, STAGE, max_block_threads(DT, OP, U, STAGE)))
    k_reduce(const KParams p) {
  using T = Tr<DT, OP>;
  using Acc = typename T::Acc;
  // Programmatic dependent launch: this grid may be resident before the
  // previous kernel of the stream has finished; nothing is read or written
  // before the dependency resolves.  The next kernel may be scheduled once
  // every block has triggered: in a many-wave grid the last wave triggers at
  // its start (the next grid fills SMs as this one drains); in a one-wave or
  // persistent grid every block triggers after its main loop (triggering at
  // the start would park the next grid's CTAs on the SMs for the whole run).
  // A team call whose members share this GPU never triggers: the next grid's
  // parked CTAs could fill the SMs a co-resident member needs to reach the
  // exchange this grid's last block is waiting in.
  // Before the dependency resolves only the input is touched, in one of two ways:
  //  * p.early == 2 (default): thread 0 issues one bulk L2 prefetch of the
  //    block's first tile -- a hint with no effect on memory consistency, so it
  //    is correct whoever writes the input and whenever; the bytes stream into
  //    L2 during the previous grid's drain and the loads after the wait hit L2.
  //  * p.early == 1 (REDUCE_FLAG_INPUT_READY, the caller guarantees no running
  //    kernel writes the input, and it is not the previous library output): a
  //    block that is resident before the dependency resolves loads its first
  //    tile into registers, and folds it after the wait (same order, same
  //    numerics).  (U <= 4 only: with 8 loads per thread the prefetched
  //    registers would be allocated beside the loop's -- 94 -> 120 registers,
  //    one block less per SM; the U = 8 kernels prefetch into L2 instead.)
  constexpr bool kEarly = STAGE == STAGE_REG && U <= 4;
  uint32_t pre[kEarly ? U : 1][8];
  bool have_pre = false;
  if constexpr (kEarly) {
    const long long tv = (long long)blockDim.x * U;
    if (p.early == 1 && (long long)blockIdx.x < p.tiles && (unsigned long long)((blockIdx.x + 1) * tv) <= p.body_vecs) {
      const char* ptr = p.body + ((unsigned long long)(blockIdx.x * tv) + threadIdx.x) * kVecBytes;
#pragma unroll
      for (int u = 0; u < U; ++u) ld_v8(ptr + (size_t)u * blockDim.x * kVecBytes, pre[u]);
      have_pre = true;
    }
  }
  if (p.early != 0 && threadIdx.x == 0 && (int)blockIdx.x < p.pf_stride) {
    // bulk L2 prefetches of the tiles this block (and, when the grid has more
    // blocks than fit at once, the blocks of later waves) will read: the HBM
    // reads run while the previous grid drains; the loads after the wait hit L2
    const unsigned long long tv = (unsigned long long)blockDim.x * U;
    long long t = blockIdx.x + (have_pre ? p.pf_stride : 0);
#pragma unroll 1
    for (int k = have_pre ? 1 : 0; k < p.pf_tiles && t < p.tiles; ++k, t += p.pf_stride) {
      const unsigned long long v0 = (unsigned long long)t * tv;
      const unsigned long long nv = v0 + tv <= p.body_vecs ? tv : p.body_vecs - v0;
      prefetch_l2_bulk(p.body + v0 * kVecBytes, (uint32_t)(nv * kVecBytes));
    }
  }
  pdl_wait();
  const bool may_trigger = !p.team.shared_gpu;
  const unsigned win = p.trig_window;
  const bool early_trigger = may_trigger && gridDim.x > win && blockIdx.x + win >= gridDim.x;
  if (early_trigger) pdl_trigger();
  if (p.gc == GC_CLUSTER) cluster_arrive_relaxed();  // phase 1: "this CTA has started"
  // GC_FLAGS: this call's epoch, read now so the load's latency hides behind the tiles
  const unsigned ep = (p.gc == GC_FLAGS && threadIdx.x == 0) ? ld_relaxed_u32(p.ticket) + 1u : 0u;
  Part<T> a[T::NA];
  init_parts<T>(a);
  uint32_t aux = 0;

  const long long B = blockDim.x;
  const long long tile_vecs = B * U;
  long long tile_first = blockIdx.x;
  if constexpr (kEarly) {
    if (have_pre) {
#pragma unroll
      for (int u = 0; u < U; ++u) fold_vec<T>(a, aux, pre[u], u);
      tile_first += gridDim.x;
    }
  }

  // no unrolling: an unrolled loop makes the compiler compute the trip count
  // with a 64-bit division (a CALL to the division routine) in every block's
  // prologue -- measurable latency at medium sizes, where the default grid
  // runs this loop exactly once
#pragma unroll 1
  for (long long tile = tile_first; tile < p.tiles; tile += gridDim.x) {
    const unsigned long long v0 = (unsigned long long)(tile * tile_vecs) + threadIdx.x;
    const char* ptr = p.body + v0 * kVecBytes;
    const bool full = (unsigned long long)((tile + 1) * tile_vecs) <= p.body_vecs;
    if constexpr (STAGE == STAGE_SMEM) {
      // Each thread stages exactly the vectors it will fold (vector v0 + u*B
      // -> slot u*B + t), so no block barrier is needed: cp.async.wait_all
      // waits for this thread's own copies.  All 2U copies are in flight at once.
      extern __shared__ __align__(128) unsigned char stile[];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (full || v0 + (unsigned long long)(u * B) < p.body_vecs) {
          unsigned char* d = stile + ((size_t)u * B + threadIdx.x) * kVecBytes;
          const char* g = ptr + (size_t)u * B * kVecBytes;
          cp_async16(d, g);
          cp_async16(d + 16, g + 16);
        }
      }
      cp_async_wait_all();
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (full || v0 + (unsigned long long)(u * B) < p.body_vecs) {
          uint32_t r[8];
          lds_v8(stile + ((size_t)u * B + threadIdx.x) * kVecBytes, r);
          fold_vec<T>(a, aux, r, u);
        }
      }
    } else if (full) {
      uint32_t r[U][8];
#pragma unroll
      for (int u = 0; u < U; ++u) ld_v8(ptr + (size_t)u * B * kVecBytes, r[u]);
#pragma unroll
      for (int u = 0; u < U; ++u) fold_vec<T>(a, aux, r[u], u);
    } else {  // the ragged last tile
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (v0 + (unsigned long long)(u * B) < p.body_vecs) {
          uint32_t r[8];
          ld_v8(ptr + (size_t)u * B * kVecBytes, r);
          fold_vec<T>(a, aux, r, u);
        }
      }
    }
  }
  if (may_trigger && !early_trigger && gridDim.x <= win) pdl_trigger();
  if (blockIdx.x == gridDim.x - 1) {
    using Elem = typename T::Elem;
    const int t = threadIdx.x;
    if (t < p.head) fold_elem<T>(a[0], aux, __ldg((const Elem*)p.in + t));
    else if (t >= 8 && t - 8 < p.tail)
      fold_elem<T>(a[0], aux, __ldg((const Elem*)(p.body + p.body_vecs * kVecBytes) + (t - 8)));
  }
  const Acc v = thread_result<T>(a, aux);
  const typename T::Grid g = block_combine<T, BC>(v);
  grid_combine<T>(g, p, ep);
}

// Second pass of GC_TWO_PASS and the cross-chunk / cross-rank combine.
template <int DT, int OP>
__global__ void __launch_bounds__(1024) k_combine(const void* vals, long long count, void* out, int raw_out,
                                                 TeamArgs team) {
  using T = Tr<DT, OP>;
  pdl_wait();
  typename T::Grid x = reduce_grid_values<T>((const typename T::Grid*)vals, count);
  if (threadIdx.x == 0) {
    if (team.k > 0) x = RB_CROSS_RANK(T, x, team);
    if (raw_out) *(typename T::Grid*)out = x;
    else T::finalize(x, out);
  }
}

template <int DT, int OP>
__global__ void k_init_slots(void* slots, unsigned* ticket) {
  using T = Tr<DT, OP>;
  if (threadIdx.x < kMaxSlots) {
    unsigned long long* w = (unsigned long long*)((char*)slots + threadIdx.x * kSlotBytes);
    w[0] = 0ull;  // the packed int32-sum word is 8 bytes wide; Grid values are <= 16
    w[1] = 0ull;
    *(typename T::Grid*)w = T::gident();
  }
  if (threadIdx.x == 0) *ticket = 0u;
}

inline KParams make_params(const LaunchDesc& d) {
  KParams p;
  p.in = (const char*)d.in;
  p.body = (const char*)d.body;
  p.body_vecs = d.body_vecs;
  p.tiles = d.tiles;
  p.head = d.head;
  p.tail = d.tail;
  p.out = d.out;
  p.raw_out = d.raw_out;
  p.gc = d.gc;
  p.slots = d.slots;
  p.nslots = d.nslots < 1 ? 1 : d.nslots;
  p.ticket = d.ticket;
  p.partials = d.partials;
  p.team = d.team;
  p.early = d.early;
  p.pf_stride = p.pf_tiles = 0;
  p.trig_window = 0;
  // TWO_PASS: the exchange happens in the second kernel, not per block
  if (d.gc == GC_TWO_PASS) p.team.k = 0;
  return p;
}

// Function attributes belong to each device's instance of the module: opt a
// kernel in to at least `smem_bytes` of dynamic shared memory (and, if asked,
// to non-portable cluster sizes).  The attribute is a maximum, so it is only
// ever raised: a later, smaller request must not undercut an earlier size.
inline cudaError_t opt_in_smem(const void* kern, int smem_bytes, bool nonportable_cluster = false) {
  static std::mutex mu;
  static std::map<std::pair<int, const void*>, int> granted;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(mu);
  const auto key = std::make_pair(dev, kern);
  auto it = granted.find(key);
  if (it != granted.end() && it->second >= smem_bytes) return cudaSuccess;
  cudaError_t e = cudaSuccess;
  if (nonportable_cluster) e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e == cudaSuccess) granted[key] = smem_bytes;
  return e;
}

// Resident blocks per SM of (kernel, block size, dynamic shared memory) on the
// current device (at least 1), computed once per (device, kernel, shape).
inline int blocks_per_sm(const void* kern, int block, size_t smem) {
  static std::mutex mu;
  static std::map<std::tuple<int, const void*, int, size_t>, int> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(mu);
  const auto key = std::make_tuple(dev, kern, block, smem);
  auto it = cache.find(key);
  if (it != cache.end()) return it->second;
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, block, smem) != cudaSuccess || nb < 1) {
    cudaGetLastError();
    nb = 1;
  }
  cache[key] = nb;
  return nb;
}

// SM count of the current device, cached per device.
inline int num_sms_cached() {
  static std::mutex mu;
  static std::map<int, int> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(dev);
  if (it != cache.end()) return it->second;
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms < 1) {
    cudaGetLastError();
    sms = 148;
  }
  cache[dev] = sms;
  return sms;
}

// Launch one k_reduce instantiation; GC_CLUSTER launches exactly one cluster
// of d.grid CTAs (sizes above the portable 8 need the non-portable opt-in);
// STAGE_SMEM needs block*U*32 bytes of dynamic shared memory (opt-in above 48 KB).
inline cudaError_t launch_kernel(void (*kern)(const KParams), const LaunchDesc& d, const KParams& p, cudaStream_t s) {
  const size_t smem = d.stage == STAGE_SMEM ? (size_t)d.block * d.unroll * kVecBytes : 0;
  // any dynamic tile opts in (static scratch + a 32 KB tile can already pass the 48 KB default)
  if (smem > 0 || (d.gc == GC_CLUSTER && d.grid > 8)) {
    const cudaError_t e = opt_in_smem((const void*)kern, kMaxSmemTileBytes, true);
    if (e != cudaSuccess) return e;
  }
  KParams q = p;
  q.pf_stride = 0;
  q.pf_tiles = 0;
  q.trig_window = kPdlBlocksPerSm * (unsigned)num_sms_cached();
  if (p.early != 0 && d.tiles > 0 && prefetch_budget_bytes() == 0) {
    // the default: every block prefetches (or loads) its own first tile only
    q.pf_stride = d.grid;
    q.pf_tiles = 1;
  } else if (p.early != 0 && d.tiles > 0) {
    // blocks resident at once (one wave): they issue the prefetches, striding
    // over the tiles, up to prefetch_budget_bytes() (L2 is 126 MB; the previous
    // grid's and this grid's streams share it)
    const long long wave = (long long)blocks_per_sm((const void*)kern, d.block, smem) * num_sms_cached();
    const long long stride = d.grid < wave ? d.grid : wave;
    const long long tile_bytes = (long long)d.block * d.unroll * kVecBytes;
    long long cap = prefetch_budget_bytes() / tile_bytes;
    if (cap < stride) cap = stride;  // at least every early block's first tile
    const long long want = d.tiles < cap ? d.tiles : cap;
    q.pf_stride = (int)stride;
    q.pf_tiles = (int)((want + stride - 1) / stride);
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(d.grid, 1, 1);
  cfg.blockDim = dim3(d.block, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if (pdl_enabled()) {
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  if (d.gc == GC_CLUSTER) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = d.grid;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = 1;
    ++na;
  }
  cfg.attrs = attr;
  cfg.numAttrs = na;
  return cudaLaunchKernelEx(&cfg, kern, q);
}

// k_combine with the same programmatic-dependent-launch attribute.
template <int DT, int OP>
cudaError_t launch_combine_kernel(const void* vals, long long count, void* out, int raw_out, int block, cudaStream_t s,
                                  TeamArgs team) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(1, 1, 1);
  cfg.blockDim = dim3(block, 1, 1);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k_combine<DT, OP>, vals, count, out, raw_out, team);
}


template <int DT, int OP, int U, int STAGE>
cudaError_t launch_bc(const LaunchDesc& d, const KParams& p, cudaStream_t s) {
  if constexpr (DT == DT_F64 && OP == OP_SUMACC) {  // no shared atomics on double-double pairs
    if (d.bc == BC_SHFL) return launch_kernel(k_reduce<DT, OP, U, BC_SHFL, STAGE>, d, p, s);
    if (d.bc == BC_TREE) return launch_kernel(k_reduce<DT, OP, U, BC_TREE, STAGE>, d, p, s);
    return cudaErrorInvalidValue;
  }
  switch (d.bc) {
    case BC_SHFL: return launch_kernel(k_reduce<DT, OP, U, BC_SHFL, STAGE>, d, p, s);
    case BC_ATOMIC_WARP: return launch_kernel(k_reduce<DT, OP, U, BC_ATOMIC_WARP, STAGE>, d, p, s);
    case BC_ATOMIC_ALL: return launch_kernel(k_reduce<DT, OP, U, BC_ATOMIC_ALL, STAGE>, d, p, s);
    case BC_TREE: return launch_kernel(k_reduce<DT, OP, U, BC_TREE, STAGE>, d, p, s);
  }
  return cudaErrorInvalidValue;
}

template <int DT, int OP>
cudaError_t launch_op(const LaunchDesc& d, cudaStream_t s) {
  const KParams p = make_params(d);
  cudaError_t e;
  if (d.stage == STAGE_SMEM) {
    switch (d.unroll) {
      case 4: e = launch_bc<DT, OP, 4, STAGE_SMEM>(d, p, s); break;
      case 8: e = launch_bc<DT, OP, 8, STAGE_SMEM>(d, p, s); break;
      case 16: e = launch_bc<DT, OP, 16, STAGE_SMEM>(d, p, s); break;
      default: return cudaErrorInvalidValue;
    }
  } else {
    switch (d.unroll) {
      case 1: e = launch_bc<DT, OP, 1, STAGE_REG>(d, p, s); break;
      case 2: e = launch_bc<DT, OP, 2, STAGE_REG>(d, p, s); break;
      case 4: e = launch_bc<DT, OP, 4, STAGE_REG>(d, p, s); break;
      case 8: e = launch_bc<DT, OP, 8, STAGE_REG>(d, p, s); break;
      default: return cudaErrorInvalidValue;
    }
  }
  if (e != cudaSuccess || d.gc != GC_TWO_PASS) return e;
  // the second pass: one block, 4 loads in flight per thread; 256 threads up to
  // 4096 partials, else 1024
  return launch_combine_kernel<DT, OP>(d.partials, (long long)d.grid, d.out, d.raw_out, d.grid <= 4096 ? 256 : 1024, s,
                                       d.team);
}

template <int DT>
cudaError_t launch_dt(const LaunchDesc& d, cudaStream_t s) {
  switch (d.op) {
    case OP_SUM: return launch_op<DT, OP_SUM>(d, s);
    case OP_MIN: return launch_op<DT, OP_MIN>(d, s);
    case OP_MAX: return launch_op<DT, OP_MAX>(d, s);
    case OP_SUMACC:
      if constexpr (DT != DT_I32) return launch_op<DT, OP_SUMACC>(d, s);
      break;
  }
  return cudaErrorInvalidValue;
}

template <int DT>
cudaError_t combine_dt(int op, const void* vals, long long count, void* out, int raw_out, int block, cudaStream_t s,
                       TeamArgs t) {
  switch (op) {
    case OP_SUM: return launch_combine_kernel<DT, OP_SUM>(vals, count, out, raw_out, block, s, t);
    case OP_MIN: return launch_combine_kernel<DT, OP_MIN>(vals, count, out, raw_out, block, s, t);
    case OP_MAX: return launch_combine_kernel<DT, OP_MAX>(vals, count, out, raw_out, block, s, t);
    case OP_SUMACC:
      if constexpr (DT != DT_I32) return launch_combine_kernel<DT, OP_SUMACC>(vals, count, out, raw_out, block, s, t);
      break;
  }
  return cudaErrorInvalidValue;
}

template <int DT>
cudaError_t init_dt(char* slots_base, char* tickets_base, cudaStream_t s) {
  k_init_slots<DT, OP_SUM><<<1, 32, 0, s>>>(slots_base + combo_index(DT, OP_SUM) * kSlotRegionBytes,
                                             (unsigned*)(tickets_base + combo_index(DT, OP_SUM) * kSlotBytes));
  k_init_slots<DT, OP_MIN><<<1, 32, 0, s>>>(slots_base + combo_index(DT, OP_MIN) * kSlotRegionBytes,
                                             (unsigned*)(tickets_base + combo_index(DT, OP_MIN) * kSlotBytes));
  k_init_slots<DT, OP_MAX><<<1, 32, 0, s>>>(slots_base + combo_index(DT, OP_MAX) * kSlotRegionBytes,
                                             (unsigned*)(tickets_base + combo_index(DT, OP_MAX) * kSlotBytes));
  if constexpr (DT != DT_I32)
    k_init_slots<DT, OP_SUMACC><<<1, 32, 0, s>>>(slots_base + combo_index(DT, OP_SUMACC) * kSlotRegionBytes,
                                                  (unsigned*)(tickets_base + combo_index(DT, OP_SUMACC) * kSlotBytes));
  return cudaPeekAtLastError();
}

}  // namespace rb
