// reduce_internal.h -- interface between the host runtime (reduce_api.cpp,
// reduce_multi.cpp) and the kernel translation units.  Not part of the ABI.
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace rb {

constexpr int kSlotBytes = 256;  // stride between global accumulator slots (separate L2 lines)
constexpr int kMaxSlots = 32;

// How a tile reaches the registers (step S2):
//   STAGE_REG  : 256-bit LDG straight into registers (U loads per thread);
//   STAGE_SMEM : cp.async (LDGSTS) 16-byte copies into a per-block shared
//                tile, then 128-bit shared loads -- the bytes in flight are not
//                bounded by registers, so a block can keep 64 KB in flight.
// Both fold the same vectors in the same order (identical numerics).
constexpr int STAGE_REG = 1, STAGE_SMEM = 2;
constexpr int kMaxSmemTileBytes = 128 * 1024;

// Largest block the (dtype, op, unroll, stage) instantiation is compiled for:
// with register staging, the budget of 64 registers/thread at 1024 threads is
// too small for 8 in-flight 32-byte loads, and for the fp64 min/max
// select+NaN-flag fold at unroll >= 2.
// Minimum resident blocks requested from ptxas for the small-unroll register
// instantiations: at 2048 threads per SM this caps them at 32 registers, i.e.
// full occupancy (the mid-size regime is latency-bound: 8 x 256-thread blocks
// keep 33 % more bytes in flight than the 6 blocks 35-36 registers allow).
constexpr int min_blocks_hint(int dtype, int op, int unroll, int stage, int max_threads) {
  return (stage == STAGE_REG && (unroll == 1 || (unroll == 2 && dtype != 0)) && op != 3 && !(dtype == 2 && op != 0))
             ? 2048 / max_threads
             // fp64 min/max: left alone, ptxas spends 96 registers at U = 4
             // (2 blocks of 256 per SM, 24 % occupancy, 3.4 TB/s one tile per
             // block); capped at 64 the loop keeps its loads in flight
             : (stage == STAGE_REG && dtype == 2 && (op == 1 || op == 2) && unroll <= 4) ? 1024 / max_threads : 1;
}

constexpr int max_block_threads(int dtype, int op, int unroll, int stage = STAGE_REG) {
  return stage == STAGE_SMEM ? (op == 3 ? 512 : 1024)
                             : ((unroll >= 8 || (dtype == 2 && op != 0 && unroll >= 2) || (op == 3 && unroll >= 4))
                                    ? 512 : 1024);
}

// Team = the ranks of a sharded reduction whose per-rank raw results are
// exchanged through peer memory inside the reduction kernel itself (SURVEY
// 8(f) N2, the "one-shot combine fused as the epilogue of the last block").
// Every rank owns one buffer of kTeamBufBytes; bufs[j] is rank j's buffer as
// seen from this GPU (a CUDA-IPC / peer mapping over NVLink, or a local pointer).
//   [0, 2*kTeamMaxRanks*32)  slots[parity][rank]: the raw value (<= 16 B) as
//                            4 pairs {word, epoch} (flag-in-data, one 8-byte access each)
//   [kTeamEpochOff, + 4)     this rank's call counter (the epoch)
// The epoch lives in device memory and is advanced by the kernel itself, so a
// team call captured in a CUDA graph stays correct on every replay.
struct TeamArgs {
  char* const* bufs;  // device array of k pointers (nullptr when not a team call)
  int k, rank;
  short shared_gpu;   // another member runs on this GPU (no early PDL trigger)
  // NVLS exchange (reduce_multi_nvls): bufs[j] is rank j's copy of an NCCL
  // symmetric window (unicast, over NVLink); bufs[k] is the window's NVLink
  // SHARP multicast address and bufs[k + 1] this member's call counters
  // ([0] LL epoch, [1] barrier calls).  nvls: 0 = the peer-store team protocol
  // above; 1 = arrive on every copy's counter with one multimem.red, then one
  // multimem.ld_reduce (the reduction happens in the NVSwitch); 2 = one
  // multimem.st of the value with the call's epoch into every copy
  // (flag-in-data), then a rank-order combine of the local copy
  // (deterministic).  (The struct keeps its 24 bytes: a larger kernel
  // parameter block cost the headline kernel 18 registers.)
  short nvls;
};
constexpr int kTeamMaxRanks = 256;
constexpr size_t kTeamSlotBytes = 32;
constexpr size_t kTeamEpochOff = 2 * kTeamMaxRanks * kTeamSlotBytes;
constexpr size_t kTeamBufBytes = kTeamEpochOff + 16;
// NVLS window layout (every rank's copy alike)
constexpr size_t kNvlsCtrOff = 0;      // u32 barrier counter (+k per call, never reset)
constexpr size_t kNvlsRedOff = 128;    // [parity] 16-byte value slots read by multimem.ld_reduce
constexpr size_t kNvlsLLOff = 4096;    // [parity][rank] 32-byte {word, epoch} pair slots
constexpr size_t kNvlsBytes = kNvlsLLOff + 2 * kTeamMaxRanks * kTeamSlotBytes;
constexpr size_t kNvlsAllocBytes = (size_t)2 << 20;  // the multicast granularity

// One launch of the main reduction kernel (steps S2-S5), fully resolved by the
// host dispatcher (step S0).
struct LaunchDesc {
  int dtype, op;
  const void* in;                // original input pointer (element-aligned)
  const void* body;              // first 32-byte-aligned element of the body
  unsigned long long body_vecs;  // 32-byte vectors in the body
  long long tiles;               // ceil(body_vecs / (block*unroll))
  int head, tail;                // scalar elements before / after the body
  int grid, block, unroll, bc, gc, stage;
  void* out;                     // device scalar (T, or the raw Grid type)
  int raw_out;                   // 1: write the un-finalised Grid value
  void* slots;                   // this (dtype, op)'s accumulator slots (GC_ATOMIC)
  int nslots;
  unsigned* ticket;              // this (dtype, op)'s ticket (GC_ATOMIC / GC_LAST_BLOCK)
  void* partials;                // Grid[grid] (GC_TWO_PASS / GC_LAST_BLOCK)
  TeamArgs team;                 // team.k > 0: exchange the raw result with the team first
  int early;                     // before griddepcontrol.wait: 1 = load the first tile into registers
                                 // (REDUCE_FLAG_INPUT_READY, input not the previous library output),
                                 // 2 = bulk L2 prefetch of the first tile (a hint, always correct)
};

// Long-segment queue of a segmented call (lives in the stream's workspace):
// segments too long for one group are cut into chunks that whole blocks reduce
// (k_seg_chunks), then their chunk partials are combined in order (k_seg_finish).
constexpr unsigned kSegQItems = 1u << 18;  // chunk items (and partial slots)
constexpr unsigned kSegQLongs = 1u << 17;  // long segments (each uses >= 2 items)
constexpr size_t kSegQHdrBytes = 256;
constexpr size_t kSegQBytes = kSegQHdrBytes + (size_t)kSegQItems * 16 /* items */ +
                              (size_t)kSegQItems * 16 /* partials */ + (size_t)kSegQLongs * 24 /* longs */;
struct SegQueue {
  unsigned* hdr;       // [0] items reserved, [1] long segments, [2] finish ticket (self-resetting)
  long long* items;    // [2 * i]: chunk i = elements [lo, hi)
  void* partials;      // Grid[kSegQItems]: chunk i's value
  long long* longs;    // [3 * j]: segment, first partial, partial count
};
inline SegQueue seg_queue_at(char* base) {
  SegQueue q;
  q.hdr = (unsigned*)base;
  q.items = (long long*)(base + kSegQHdrBytes);
  q.partials = base + kSegQHdrBytes + (size_t)kSegQItems * 16;
  q.longs = (long long*)(base + kSegQHdrBytes + (size_t)kSegQItems * 32);
  return q;
}

// Element-balanced segmented reduction of an offsets array (reduce_segbal.cuh):
// the elements are cut into fixed 4 KB chunks and every warp of a one-wave
// grid reduces one contiguous range of chunks whatever the segment lengths;
// the pieces of segments that cross ranges are joined by a fix-up pass.
constexpr unsigned kBalRanges = 1u << 16;  // capacity of the per-range arrays (ranges = chunk-kernel warps)
constexpr size_t kBalHdrBytes = 256;
constexpr size_t kBalBytes = kBalHdrBytes + (size_t)kBalRanges * (4 /* start_seg */ + 16 /* first */ +
                                                                   16 /* last */ + 4 /* last_seg */ + 4 /* flags */);
struct SegBal {
  unsigned* hdr;         // [0] non-monotone offsets seen (set by the scan, cleared by the fix-up kernel)
  unsigned* start_seg;   // [w]: the segment holding range w's first element
  void* first_val;       // Grid[w]: range w's piece of the segment open at its start
  void* last_val;        // Grid[w]: range w's piece of the segment still open at its end
  unsigned* last_seg;    // [w]: that open segment (0xFFFFFFFF: none)
  unsigned* flags;       // [w]: 1 if a segment boundary lies inside range w
  long long nranges;     // ranges = warps of the chunk kernel's grid (set by the launcher)
};
inline SegBal seg_bal_at(char* base) {
  SegBal b;
  char* p = base + kBalHdrBytes;
  b.hdr = (unsigned*)base;
  b.first_val = p;  p += (size_t)kBalRanges * 16;
  b.last_val = p;   p += (size_t)kBalRanges * 16;
  b.start_seg = (unsigned*)p;  p += (size_t)kBalRanges * 4;
  b.last_seg = (unsigned*)p;   p += (size_t)kBalRanges * 4;
  b.flags = (unsigned*)p;
  b.nranges = 0;
  return b;
}

// One segmented / batched call, see reduce_segmented.cuh.
struct SegParams {
  const char* in;
  const long long* offsets;  // device, nseg + 1 entries; NULL: uniform segments of seg_len
  long long seg_len;
  long long nseg;
  void* out;                 // T[nseg] (finalised) or Grid[nseg] (raw)
  int raw_out;
  int use_q;                 // 1: offload long segments to q (2 more launches)
  int tail;                  // 1: fold a segment's last vectors in one predicated round
  SegQueue q;
  int rows_nv;               // > 0: uniform 32-byte-aligned rows of rows_nv (<= 8) vectors, one
                             //      thread per row with all its loads in flight (k_rows_aligned)
  int rows_tiled;            // 6 + LV > 0: uniform 32-byte-aligned rows of 32 << LV vectors
                             //      (LV = -5..5: 32 B-32 KB), the flat tile walk (k_rows_tiled)
  long long rows_tiled_vecs; // > 0 (with rows_tiled > 0): rows of this many vectors, a multiple
                             //      of 1024 (32 KB tiles), one block per row (k_rows_tiled_big)
  int balanced;              // 1: element-balanced chunks (offsets arrays, reduce_segbal.cuh)
  SegBal b;
};
// group: lanes per segment (1, 8 or 32) or 0 = one block per segment.
cudaError_t launch_segmented(int dtype, int op, const SegParams& p, int group, int block, cudaStream_t s);

// One histogram launch, see reduce_histogram.cuh.
struct HistParams {
  const char* in;               // element-aligned input (4-byte elements)
  const char* body;             // first 32-byte-aligned element
  unsigned long long body_vecs;
  int head, tail;
  long long lo_i, hi_i;         // int32 input: integer bounds
  unsigned long long range_i;   //   hi_i - lo_i
  unsigned long long magic;     //   floor((2^64 - 1) / range_i): quotient by multiply-high
  unsigned magic32;             //   narrow: Granlund-Montgomery multiplier of range_i (exact
  int shift32;                  //   floor(n / range_i) for every 32-bit n, no correction step)
  int narrow;                   //   range_i * nbins < 2^32 (and [lo, hi) meets the int32 range):
                                //   32-bit range check and quotient
  unsigned lo_c32, lim32;       //   narrow: counted iff (uint32)(x - lo_c32) <= lim32, with [lo_c, hi_c)
                                //   = [lo, hi) clamped to the int32 range, lim32 = hi_c - 1 - lo_c
  unsigned lo32;                //   narrow: (uint32)lo_i (x - lo mod 2^32 is exact for counted x)
  float lo_f, hi_f, scale_f;    // fp32 input: (float)lo, (float)hi, (float)(nbins / (hi - lo))
  int nbins;
  unsigned* counts;             // device, nbins
  int merge64;                  // counts 8-byte aligned and n < 2^32: a bin pair is merged with ONE
                                //   64-bit global add (no count can carry into its neighbour)
};
cudaError_t launch_histogram(int dtype, const HistParams& p, int block, cudaStream_t s);

// Size in bytes of the Grid (cross-block) type of (dtype, op).
int grid_value_bytes(int dtype, int op);

cudaError_t launch_reduce(const LaunchDesc& d, cudaStream_t s);

// Reduce `count` Grid-typed values in a fixed order with one block of
// `block` threads and write the finalised (or raw) result to `out`.
cudaError_t launch_combine(int dtype, int op, const void* vals, long long count, void* out,
                           int raw_out, int block, cudaStream_t s, TeamArgs team = TeamArgs{nullptr, 0, 0, 0, 0});

// Write the identity into every accumulator slot of every (dtype, op) and zero
// the tickets.  slots_base: 9 regions of kMaxSlots*kSlotBytes; tickets: 9 words
// spaced kSlotBytes apart.
cudaError_t launch_init_workspace(void* slots_base, void* tickets_base, cudaStream_t s);

// Programmatic dependent launch of the library's kernels (default on; the
// environment variable REDUCE_NO_PDL=1 turns it off, for A/B measurements).
bool pdl_enabled();
// Touching the input before the programmatic dependency resolves at all
// (default on; REDUCE_NO_EARLY=1 turns both forms off, for A/B measurements).
bool early_enabled();
// The bulk L2 prefetch of a block's first tile before the wait (default on;
// REDUCE_NO_PREFETCH=1 turns it off).
bool prefetch_enabled();
// Bytes a grid prefetches into L2 before its dependency resolves (at least
// every early-resident block's first tile); REDUCE_PREFETCH_MB, default 0 (first tiles only).
long long prefetch_budget_bytes();
// REDUCE_NO_ROWS_TILED=1: reduce_batched's auto choice skips k_rows_tiled
bool rows_tiled_enabled();

constexpr int kCombos = 12;  // 3 dtypes x 4 ops (sum, min, max, accurate sum)
constexpr int combo_index(int dtype, int op) { return dtype * 4 + op; }
constexpr size_t kSlotRegionBytes = (size_t)kMaxSlots * kSlotBytes;

}  // namespace rb
