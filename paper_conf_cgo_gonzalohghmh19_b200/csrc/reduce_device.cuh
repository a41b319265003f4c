// reduce_device.cuh -- device-side building blocks of the B200 reduction path.
//
// Element / accumulator traits per (dtype, op), the 32-byte streaming load, the
// warp combine (step S3), the four block combines (step S4) and the grid
// combines (step S5).  Citations P:Lnnn are PAPER.md lines (the CGO'19 paper);
// section numbers are DESIGN.md's.
//
// Hardware facts this file relies on (measured on the B200, see
// profiles/r01_probe_sm100.txt):
//   * FMNMX / DSETP.MAX order -0.0 < +0.0, and `max.NaN.f32` / `min.NaN.f32`
//     return the canonical NaN 0x7FFFFFFF whenever an input is NaN;
//   * `redux.sync.{min,max}.NaN.f32` (CREDUX.*.F32.NAN) has the same semantics;
//   * `ld.global.nc.L1::no_allocate.v8` is a single 256-bit LDG (sm_100 only).
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>
#include "reduce_internal.h"

namespace rb {

constexpr int DT_I32 = 0, DT_F32 = 1, DT_F64 = 2;
constexpr int OP_SUM = 0, OP_MIN = 1, OP_MAX = 2, OP_SUMACC = 3;
constexpr int BC_SHFL = 0, BC_ATOMIC_WARP = 1, BC_ATOMIC_ALL = 2, BC_TREE = 3;
constexpr int GC_DIRECT = 0, GC_ATOMIC = 1, GC_TWO_PASS = 2, GC_LAST_BLOCK = 3, GC_CLUSTER = 4, GC_FLAGS = 5;
constexpr int kVecBytes = 32;    // one 256-bit load per thread per vector

// ------------------------------------------------------------------ loads ---
// Streaming 32-byte read-only load; never allocates in L1 (each byte is read
// once).  Not `volatile`: the compiler may hoist/batch these (they read memory
// no thread writes during the kernel).
// RB_LD_HINT (A/B experiment hook: REDUCE_B200_NVCC_FLAGS=-DRB_LD_HINT=k builds,
// tools/probes/lib_ab.sh + sweep_ab.py): 1 adds the 256-byte L2 prefetch-size
// hint (SASS LTC256B), 2 the L2 evict_first priority (EFL2).  Neither moves any
// size 16 KB-1 GiB by more than run-to-run noise (profiles/r01_ld_hint_ab.jsonl):
// each warp's 256-bit load already covers 1 KB of whole 256-byte sectors.
#ifndef RB_LD_HINT
#define RB_LD_HINT 0
#endif
#if RB_LD_HINT == 1
#define RB_LD_V8 "ld.global.nc.L1::no_allocate.L2::256B.v8.u32"
#elif RB_LD_HINT == 2
#define RB_LD_V8 "ld.global.nc.L1::no_allocate.L2::evict_first.v8.u32"
#else
#define RB_LD_V8 "ld.global.nc.L1::no_allocate.v8.u32"
#endif
__device__ __forceinline__ void ld_v8(const void* p, uint32_t (&r)[8]) {
  asm(RB_LD_V8 " {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
      : "l"(p));
}

// cp.async (LDGSTS): 16 bytes global -> shared, L2 only (.cg), asynchronous.
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(s), "l"(gmem) : "memory");
}
// Bulk L2 prefetch (sm_90+, UBLKPF): a hint that moves `bytes` (multiple of
// 16, 16-byte-aligned source) from HBM into L2 without touching registers or
// shared memory.  A prefetch has no effect on memory consistency, so it may be
// issued before griddepcontrol.wait: a store of the previous kernel reaching
// L2 afterwards updates the prefetched line, and the loads after the wait read
// the current data from L2.
__device__ __forceinline__ void prefetch_l2_bulk(const void* gmem, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(gmem), "r"(bytes) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
// one 32-byte vector from shared memory as 8 words
__device__ __forceinline__ void lds_v8(const void* smem, uint32_t (&r)[8]) {
  const uint4 a = reinterpret_cast<const uint4*>(smem)[0];
  const uint4 b = reinterpret_cast<const uint4*>(smem)[1];
  r[0] = a.x; r[1] = a.y; r[2] = a.z; r[3] = a.w; r[4] = b.x; r[5] = b.y; r[6] = b.z; r[7] = b.w;
}

// Programmatic dependent launch (sm_90+): wait for the preceding grid of the
// stream (a no-op when it was not launched programmatically), and let the next
// programmatic grid be scheduled.
// The trigger window (blocks of the last ~full wave) is 8 blocks per SM of the
// device the kernel runs on; the host passes it in the kernel parameters.
constexpr unsigned kPdlBlocksPerSm = 8u;
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// Ticket increment with acquire-release semantics at GPU scope: the release
// half publishes this thread's earlier stores / reductions (the block's
// partial) before the increment, the acquire half makes every earlier
// publisher's data visible to the thread that draws the last ticket.  Replaces
// __threadfence() (fence.sc.gpu) + a relaxed atomic on the combine's critical path.
__device__ __forceinline__ unsigned ticket_acq_rel(unsigned* t) {
  unsigned old;
  asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(old) : "l"(t) : "memory");
  return old;
}

// Relaxed GPU-scope accesses of the flag-in-data partial records (GC_FLAGS):
// served by L2, never by a stale L1 line.
__device__ __forceinline__ unsigned ld_relaxed_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_u32(unsigned* p, unsigned v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_pairs_gpu(void* p, unsigned a, unsigned b, unsigned e) {
  asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1, %2, %3, %4};" :: "l"(p), "r"(a), "r"(e), "r"(b), "r"(e)
               : "memory");
}
__device__ __forceinline__ uint4 ld_pairs_gpu(const void* p) {
  uint4 v;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p) : "memory");
  return v;
}

// Split cluster barrier (all threads of every CTA of the cluster take part).
__device__ __forceinline__ void cluster_arrive_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() { asm volatile("barrier.cluster.wait.aligned;" ::: "memory"); }

// ------------------------------------------------------- fp primitives ---
__device__ __forceinline__ float fmax_nan(float a, float b) {
  float r; asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r;
}
__device__ __forceinline__ float fmin_nan(float a, float b) {
  float r; asm("min.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r;
}
__device__ __forceinline__ float redux_max_nan(float a) {
  float r; asm("redux.sync.max.NaN.f32 %0, %1, 0xffffffff;" : "=f"(r) : "f"(a)); return r;
}
__device__ __forceinline__ float redux_min_nan(float a) {
  float r; asm("redux.sync.min.NaN.f32 %0, %1, 0xffffffff;" : "=f"(r) : "f"(a)); return r;
}
// fp64 min/max: max.f64 is sign-aware but drops NaN; NaN is tracked separately
// in the streaming loop and re-applied here for the combine trees.
__device__ __forceinline__ double dmax_sel(double a, double b) {
  double r; asm("max.f64 %0, %1, %2;" : "=d"(r) : "d"(a), "d"(b)); return r;
}
__device__ __forceinline__ double dmin_sel(double a, double b) {
  double r; asm("min.f64 %0, %1, %2;" : "=d"(r) : "d"(a), "d"(b)); return r;
}
// 1 iff a or b is NaN (one unordered compare for two elements)
__device__ __forceinline__ uint32_t dnan2(double a, double b) {
  uint32_t r;
  asm("{\n\t.reg .pred p;\n\tsetp.nan.f64 p, %1, %2;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(r) : "d"(a), "d"(b));
  return r;
}
__device__ __forceinline__ double nan64() { return __longlong_as_double(0x7FF8000000000000ll); }

// Order-preserving keys (reading R3): unsigned order of key(x) == the order
// -inf < ... < -0.0 < +0.0 < ... < +inf, and NaN maps to the extreme that wins
// for the op (0 for min, all-ones for max), so integer min/max atomics give the
// exact fp min/max with NaN propagation.  Decoding the winning sentinel yields
// the canonical quiet NaN.
template <bool kMax>
__device__ __forceinline__ uint32_t key32(float x) {
  uint32_t b = __float_as_uint(x);
  if (x != x) return kMax ? 0xFFFFFFFFu : 0u;
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
template <bool kMax>
__device__ __forceinline__ uint32_t unkey32(uint32_t k) {
  if (kMax ? (k == 0xFFFFFFFFu) : (k == 0u)) return 0x7FC00000u;
  return (k & 0x80000000u) ? (k & 0x7FFFFFFFu) : ~k;
}
template <bool kMax>
__device__ __forceinline__ unsigned long long key64(double x) {
  unsigned long long b = (unsigned long long)__double_as_longlong(x);
  if (x != x) return kMax ? ~0ull : 0ull;
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
template <bool kMax>
__device__ __forceinline__ unsigned long long unkey64(unsigned long long k) {
  if (kMax ? (k == ~0ull) : (k == 0ull)) return 0x7FF8000000000000ull;
  return (k >> 63) ? (k & 0x7FFFFFFFFFFFFFFFull) : ~k;
}

// Butterfly exchange for scalar types and for double2 (double-double pairs).
template <class V>
__device__ __forceinline__ V shfl_xor(V v, int o) { return __shfl_xor_sync(0xffffffffu, v, o); }
__device__ __forceinline__ double2 shfl_xor(double2 v, int o) {
  return make_double2(__shfl_xor_sync(0xffffffffu, v.x, o), __shfl_xor_sync(0xffffffffu, v.y, o));
}

// Generic butterfly with a combine functor; result in all lanes.
template <class V, class F>
__device__ __forceinline__ V warp_butterfly(V v, F f) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = f(v, shfl_xor(v, o));
  return v;
}

// ------------------------------------------------------------- traits ---
// Acc  : per-thread / warp / block value;  NA independent accumulators per thread.
// Grid : type of the cross-block combine (atomics, partials, raw output).
// fold(a, aux, x): a (+)= x for one element; aux carries fp64 NaN flags.
template <int DT, int OP> struct Tr;

template <int OP> struct TrI32 {
  static constexpr int kOp = OP;
  using Elem = int32_t;
  using Acc = typename std::conditional<OP == OP_SUM, uint32_t, int32_t>::type;
  using Grid = Acc;
  static constexpr int VE = 8, NA = 2, kLaneWords = 1;
  static constexpr bool kVecTree = true;
  // The ATOMIC grid combine of int32 sums carries value and ticket in ONE
  // 64-bit atomic add (grid_combine): no fence, no second round trip.
  static constexpr bool kPackedTicket = OP == OP_SUM;
  __device__ static Acc lift(uint32_t w) { return Acc(w); }
  __device__ static Acc ident() {
    return OP == OP_SUM ? Acc(0) : (OP == OP_MIN ? Acc(0x7FFFFFFF) : Acc(0x80000000));
  }
  __device__ static Acc comb(Acc a, Acc b) {
    return OP == OP_SUM ? Acc(a + b) : (OP == OP_MIN ? (a < b ? a : b) : (a > b ? a : b));
  }
  __device__ static void fold(Acc& a, uint32_t&, uint32_t w) { a = comb(a, Acc(w)); }
  __device__ static Acc warp(Acc v) {  // REDUX / CREDUX, one instruction
    if (OP == OP_SUM) return __reduce_add_sync(0xffffffffu, (unsigned)v);
    if (OP == OP_MIN) return __reduce_min_sync(0xffffffffu, (int)v);
    return __reduce_max_sync(0xffffffffu, (int)v);
  }
  __device__ static Acc finish(Acc a, uint32_t) { return a; }
  __device__ static Grid to_grid(Acc a) { return a; }
  __device__ static Grid gident() { return ident(); }
  __device__ static Grid gcomb(Grid a, Grid b) { return comb(a, b); }
  __device__ static Grid gwarp(Grid v) { return warp(v); }
  __device__ static void gred(Grid* p, Grid v) {  // global or shared (generic address)
    if (OP == OP_SUM) atomicAdd((unsigned*)p, (unsigned)v);
    else if (OP == OP_MIN) atomicMin((int*)p, (int)v);
    else atomicMax((int*)p, (int)v);
  }
  __device__ static Grid gexch(Grid* p, Grid v) { return (Grid)atomicExch((unsigned*)p, (unsigned)v); }
  __device__ static void finalize(Grid g, void* out) { *(int32_t*)out = (int32_t)g; }
};

template <int OP> struct TrF32 {
  static constexpr int kOp = OP;
  using Elem = float;
  using Acc = float;
  using Grid = typename std::conditional<OP == OP_SUM, double, uint32_t>::type;
  static constexpr int VE = 8, NA = 2, kLaneWords = 1;
  static constexpr bool kVecTree = true;
  static constexpr bool kMax = OP == OP_MAX;
  __device__ static float lift(uint32_t w) { return __uint_as_float(w); }
  __device__ static Acc ident() {
    return OP == OP_SUM ? 0.0f : (OP == OP_MIN ? __int_as_float(0x7F800000) : __int_as_float(0xFF800000));
  }
  __device__ static Acc comb(Acc a, Acc b) {
    return OP == OP_SUM ? a + b : (OP == OP_MIN ? fmin_nan(a, b) : fmax_nan(a, b));
  }
  __device__ static void fold(Acc& a, uint32_t&, uint32_t w) { a = comb(a, __uint_as_float(w)); }
  __device__ static Acc warp(Acc v) {
    if (OP == OP_MIN) return redux_min_nan(v);
    if (OP == OP_MAX) return redux_max_nan(v);
    return warp_butterfly(v, [](float x, float y) { return x + y; });
  }
  __device__ static Acc finish(Acc a, uint32_t) { return a; }
  // fp32 sums cross blocks in fp64 (accuracy at no bandwidth cost).
  __device__ static Grid to_grid(Acc a) {
    if constexpr (OP == OP_SUM) return (double)a; else return key32<kMax>(a);
  }
  __device__ static Grid gident() {
    if constexpr (OP == OP_SUM) return 0.0; else return key32<kMax>(ident());
  }
  __device__ static Grid gcomb(Grid a, Grid b) {
    if constexpr (OP == OP_SUM) return a + b; else return kMax ? (a > b ? a : b) : (a < b ? a : b);
  }
  __device__ static Grid gwarp(Grid v) {
    if constexpr (OP == OP_SUM) return warp_butterfly(v, [](double x, double y) { return x + y; });
    else return kMax ? __reduce_max_sync(0xffffffffu, v) : __reduce_min_sync(0xffffffffu, v);
  }
  __device__ static void gred(Grid* p, Grid v) {
    if constexpr (OP == OP_SUM) atomicAdd(p, v);
    else if constexpr (kMax) atomicMax(p, v);
    else atomicMin(p, v);
  }
  __device__ static Grid gexch(Grid* p, Grid v) {
    if constexpr (OP == OP_SUM)
      return __longlong_as_double((long long)atomicExch((unsigned long long*)p, (unsigned long long)__double_as_longlong(v)));
    else return atomicExch(p, v);
  }
  __device__ static void finalize(Grid g, void* out) {
    if constexpr (OP == OP_SUM) {
      float f = (float)g;
      *(uint32_t*)out = (f != f) ? 0x7FC00000u : __float_as_uint(f);
    } else {
      *(uint32_t*)out = unkey32<kMax>(g);
    }
  }
};

template <int OP> struct TrF64 {
  static constexpr int kOp = OP;
  using Elem = double;
  using Acc = double;
  using Grid = typename std::conditional<OP == OP_SUM, double, unsigned long long>::type;
  // Vector tree into 2 accumulators.  min/max (kSelNaN): the streaming tree
  // is plain compare-selects (DSETP + 2 SEL; max.f64 lowers to ~3x that with
  // its NaN quieting and register shuffles, which made the fp64 min/max loop
  // issue-bound), and what those selects get wrong is repaired per thread in
  // finish(): NaN from a sticky flag (aux bit 0, one unordered compare per two
  // elements), and the sign of a zero result from aux bit 31 -- for max "some
  // element had its sign bit clear", for min "some element had it set".  If
  // the max is +-0 every element is <= 0, so a sign-clear element can only be
  // +0 (or NaN, flagged anyway); symmetrically for min.
  static constexpr int VE = 4, NA = 2, kLaneWords = 2;
  static constexpr bool kVecTree = true;
  static constexpr bool kSelNaN = OP != OP_SUM;
  __device__ static double sel(double a, double b) { return OP == OP_MIN ? (b < a ? b : a) : (b > a ? b : a); }
  __device__ static void fold4(double& a, uint32_t& aux, const uint32_t (&r)[8]) {
    const double x0 = __hiloint2double((int)r[1], (int)r[0]), x1 = __hiloint2double((int)r[3], (int)r[2]);
    const double x2 = __hiloint2double((int)r[5], (int)r[4]), x3 = __hiloint2double((int)r[7], (int)r[6]);
    aux |= dnan2(x0, x1) | dnan2(x2, x3);
    if (OP == OP_MIN) aux |= (r[1] | r[3] | r[5] | r[7]) & 0x80000000u;
    else aux |= ~(r[1] & r[3] & r[5] & r[7]) & 0x80000000u;
    a = sel(a, sel(sel(x0, x1), sel(x2, x3)));
  }
  static constexpr bool kMax = OP == OP_MAX;
  __device__ static double lift(double x) { return x; }
  __device__ static Acc ident() {
    return OP == OP_SUM ? 0.0 : __longlong_as_double(OP == OP_MIN ? 0x7FF0000000000000ll : (long long)0xFFF0000000000000ull);
  }
  // NaN-propagating combine (trees): sign-aware select, then NaN override.
  __device__ static Acc comb(Acc a, Acc b) {
    if (OP == OP_SUM) return a + b;
    double m = OP == OP_MIN ? dmin_sel(a, b) : dmax_sel(a, b);
    return (a != a || b != b) ? nan64() : m;
  }
  // Streaming fold: select + a sticky NaN flag (cheaper than the full comb).
  __device__ static void fold(Acc& a, uint32_t& aux, double x) {
    if (OP == OP_SUM) { a += x; return; }
    a = OP == OP_MIN ? dmin_sel(a, x) : dmax_sel(a, x);
    aux |= (x != x) ? 1u : 0u;
  }
  __device__ static Acc warp(Acc v) { return warp_butterfly(v, [](double x, double y) { return comb(x, y); }); }
  __device__ static Acc finish(Acc a, uint32_t aux) {
    if (OP == OP_SUM) return a;
    if (aux & 1u) return nan64();
    if (a == 0.0 && (aux >> 31)) return OP == OP_MIN ? -0.0 : 0.0;
    return a;
  }
  __device__ static Grid to_grid(Acc a) {
    if constexpr (OP == OP_SUM) return a; else return key64<kMax>(a);
  }
  __device__ static Grid gident() {
    if constexpr (OP == OP_SUM) return 0.0; else return key64<kMax>(ident());
  }
  __device__ static Grid gcomb(Grid a, Grid b) {
    if constexpr (OP == OP_SUM) return a + b; else return kMax ? (a > b ? a : b) : (a < b ? a : b);
  }
  __device__ static Grid gwarp(Grid v) { return warp_butterfly(v, [](Grid x, Grid y) { return gcomb(x, y); }); }
  __device__ static void gred(Grid* p, Grid v) {
    if constexpr (OP == OP_SUM) atomicAdd(p, v);
    else if constexpr (kMax) atomicMax(p, v);
    else atomicMin(p, v);
  }
  __device__ static Grid gexch(Grid* p, Grid v) {
    if constexpr (OP == OP_SUM)
      return __longlong_as_double((long long)atomicExch((unsigned long long*)p, (unsigned long long)__double_as_longlong(v)));
    else return atomicExch(p, v);
  }
  __device__ static void finalize(Grid g, void* out) {
    if constexpr (OP == OP_SUM) {
      *(unsigned long long*)out = (g != g) ? 0x7FF8000000000000ull : (unsigned long long)__double_as_longlong(g);
    } else {
      *(unsigned long long*)out = unkey64<kMax>(g);
    }
  }
};

// ---- accurate sums: same bandwidth, tighter error --------
// fp32 input, fp64 accumulation from the first add: error <= u_f|S| + (L+1) u_d sum|x|.
// Per thread: Neumaier pairs (s, c) in fp32 -- FP32-pipe work only, since the
// B200's FP64 pipe cannot convert and add 2^28 elements at HBM speed -- then
// s and c are converted to fp64 once per thread (exactly) and everything above
// the thread runs in fp64.  The per-thread residual is O(n_t u_f^2) sum|x|.
struct TrF32Acc {
  static constexpr int kOp = OP_SUMACC;
  using Elem = float;
  using Acc = double;
  using Grid = double;
  using Part = float2;  // x = s, y = c
  static constexpr int VE = 8, NA = 8, kLaneWords = 1;
  static constexpr bool kVecTree = false;
  __device__ static Acc ident() { return 0.0; }
  __device__ static Part part_ident() { return make_float2(0.0f, 0.0f); }
  __device__ static Acc part_to_acc(Part p) { return isfinite(p.x) ? (double)p.x + (double)p.y : (double)p.x; }
  __device__ static Acc comb(Acc a, Acc b) { return a + b; }
  __device__ static void fold(Part& a, uint32_t&, uint32_t w) {
    const float x = __uint_as_float(w);
    const float t = a.x + x;
    const bool s_big = fabsf(a.x) >= fabsf(x);
    const float big = s_big ? a.x : x, small = s_big ? x : a.x;
    a.y += (big - t) + small;
    a.x = t;
  }
  __device__ static Acc warp(Acc v) { return warp_butterfly(v, [](double x, double y) { return x + y; }); }
  __device__ static Acc finish(Acc a, uint32_t) { return a; }
  __device__ static Grid to_grid(Acc a) { return a; }
  __device__ static Grid gident() { return 0.0; }
  __device__ static Grid gcomb(Grid a, Grid b) { return a + b; }
  __device__ static Grid gwarp(Grid v) { return warp(v); }
  __device__ static void gred(Grid* p, Grid v) { atomicAdd(p, v); }
  __device__ static Grid gexch(Grid* p, Grid v) {
    return __longlong_as_double((long long)atomicExch((unsigned long long*)p, (unsigned long long)__double_as_longlong(v)));
  }
  __device__ static void finalize(Grid g, void* out) {
    const float f = (float)g;
    *(uint32_t*)out = (f != f) ? 0x7FC00000u : __float_as_uint(f);
  }
};

// fp64 input, double-double accumulation: each accumulator is (hi, lo) with
// Neumaier's fold (Neumaier 1974) and Knuth's TwoSum for merging pairs; the
// result is hi + lo rounded once.  Non-finite inputs are carried by hi alone
// (hi is the plain running sum), so inf / NaN follow reading R2.
struct TrF64Acc {
  static constexpr int kOp = OP_SUMACC;
  using Elem = double;
  using Acc = double2;  // x = hi, y = lo
  using Grid = double2;
  static constexpr int VE = 4, NA = 4, kLaneWords = 2;
  static constexpr bool kVecTree = false;
  __device__ static Acc ident() { return make_double2(0.0, 0.0); }
  __device__ static Acc comb(Acc a, Acc b) {
    const double s = a.x + b.x;                       // TwoSum(a.hi, b.hi)
    const double bb = s - a.x;
    const double e = (a.x - (s - bb)) + (b.x - bb);
    const double lo = a.y + b.y + e;
    const double hi = s + lo;                         // FastTwoSum renormalise
    return make_double2(isfinite(s) ? hi : s, isfinite(s) ? lo - (hi - s) : 0.0);
  }
  __device__ static void fold(Acc& a, uint32_t&, double x) {
    const double t = a.x + x;
    a.y += (fabs(a.x) >= fabs(x)) ? (a.x - t) + x : (x - t) + a.x;
    a.x = t;
  }
  __device__ static Acc warp(Acc v) { return warp_butterfly(v, [](double2 x, double2 y) { return comb(x, y); }); }
  __device__ static Acc finish(Acc a, uint32_t) { return a; }
  __device__ static Grid to_grid(Acc a) { return a; }
  __device__ static Grid gident() { return ident(); }
  __device__ static Grid gcomb(Grid a, Grid b) { return comb(a, b); }
  __device__ static Grid gwarp(Grid v) { return warp(v); }
  __device__ static void gred(Grid*, Grid) { __trap(); }        // no 128-bit fp atomics: ATOMIC is never planned
  __device__ static Grid gexch(Grid*, Grid) { __trap(); return ident(); }
  __device__ static void finalize(Grid g, void* out) {
    const double r = isfinite(g.x) ? g.x + g.y : g.x;
    *(unsigned long long*)out = (r != r) ? 0x7FF8000000000000ull : (unsigned long long)__double_as_longlong(r);
  }
};

template <int OP> struct Tr<DT_I32, OP> : TrI32<OP> {};
template <int OP> struct Tr<DT_F32, OP> : TrF32<OP> {};
template <int OP> struct Tr<DT_F64, OP> : TrF64<OP> {};
template <> struct Tr<DT_F32, OP_SUMACC> : TrF32Acc {};
template <> struct Tr<DT_F64, OP_SUMACC> : TrF64Acc {};

// Per-thread accumulator ("part"): the traits' Part type if it declares one
// (the fp32 accurate sum keeps Neumaier (s, c) pairs in fp32), else Acc.
template <class T, class = void> struct PartOf {
  using type = typename T::Acc;
  __device__ static type ident() { return T::ident(); }
  __device__ static typename T::Acc to_acc(type p) { return p; }
};
template <class T> struct PartOf<T, std::void_t<typename T::Part>> {
  using type = typename T::Part;
  __device__ static type ident() { return T::part_ident(); }
  __device__ static typename T::Acc to_acc(type p) { return T::part_to_acc(p); }
};
template <class T> using Part = typename PartOf<T>::type;

// Fold one 32-byte vector into the per-thread accumulators.
//   kVecTree (plain sums, min, max): the vector's lanes are reduced by a
//     pairwise tree in registers (depth log2 VE) and the result is folded into
//     accumulator `slot % NA` (NA = 2: two independent chains) -- the same
//     addition depth as one accumulator per lane, with 6 fewer live registers,
//     which keeps the small-unroll kernels at 32 registers (full occupancy).
//   fp64 min/max: the same tree of selects, NaN in the sticky flag.
//   otherwise (accurate sums): lane k folds into accumulator k.
template <class T, class = void> struct HasPackedTicket : std::false_type {};
template <class T> struct HasPackedTicket<T, std::enable_if_t<T::kPackedTicket>> : std::true_type {};

template <class T, class = void> struct HasSelNaN : std::false_type {};
template <class T> struct HasSelNaN<T, std::enable_if_t<T::kSelNaN>> : std::true_type {};

template <class T>
__device__ __forceinline__ void fold_vec(Part<T> (&a)[T::NA], uint32_t& aux, const uint32_t (&r)[8], int slot) {
  if constexpr (HasSelNaN<T>::value) {
    T::fold4(a[slot % T::NA], aux, r);
  } else if constexpr (T::kVecTree) {
    using Acc = typename T::Acc;
    Acc t;
    if constexpr (T::kLaneWords == 1) {
      const Acc t01 = T::comb(T::lift(r[0]), T::lift(r[1])), t23 = T::comb(T::lift(r[2]), T::lift(r[3]));
      const Acc t45 = T::comb(T::lift(r[4]), T::lift(r[5])), t67 = T::comb(T::lift(r[6]), T::lift(r[7]));
      t = T::comb(T::comb(t01, t23), T::comb(t45, t67));
    } else {
      const Acc t01 = T::comb(T::lift(__hiloint2double((int)r[1], (int)r[0])), T::lift(__hiloint2double((int)r[3], (int)r[2])));
      const Acc t23 = T::comb(T::lift(__hiloint2double((int)r[5], (int)r[4])), T::lift(__hiloint2double((int)r[7], (int)r[6])));
      t = T::comb(t01, t23);
    }
    a[slot % T::NA] = T::comb(a[slot % T::NA], t);
  } else if constexpr (T::kLaneWords == 1) {
#pragma unroll
    for (int k = 0; k < 8; ++k) T::fold(a[k], aux, r[k]);
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k) T::fold(a[k], aux, __hiloint2double((int)r[2 * k + 1], (int)r[2 * k]));
  }
}

template <class T>
__device__ __forceinline__ void fold_elem(Part<T>& a, uint32_t& aux, typename T::Elem e) {
  if constexpr (T::kLaneWords == 1) T::fold(a, aux, *reinterpret_cast<const uint32_t*>(&e));
  else T::fold(a, aux, e);
}

template <class T>
__device__ __forceinline__ void init_parts(Part<T> (&a)[T::NA]) {
#pragma unroll
  for (int k = 0; k < T::NA; ++k) a[k] = PartOf<T>::ident();
}

// Pairwise tree over the NA accumulators (depth log2 NA), in the Acc type.
template <class T>
__device__ __forceinline__ typename T::Acc thread_result(Part<T> (&p)[T::NA], uint32_t aux) {
  typename T::Acc a[T::NA];
#pragma unroll
  for (int k = 0; k < T::NA; ++k) a[k] = PartOf<T>::to_acc(p[k]);
#pragma unroll
  for (int w = T::NA / 2; w > 0; w >>= 1)
#pragma unroll
    for (int k = 0; k < w; ++k) a[k] = T::comb(a[k], a[k + w]);
  return T::finish(a[0], aux);
}

// ------------------------------------------------------ block combine (S4) --
// Returns the block's value as T::Grid, valid in thread 0.
template <class T, int BC>
__device__ __forceinline__ typename T::Grid block_combine(typename T::Acc v) {
  using Acc = typename T::Acc;
  using Grid = typename T::Grid;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if constexpr (BC == BC_SHFL) {
    // "Vs": warp shuffle/redux, partial[32] in shared memory, warp 0 again
    // (Listing 4 lines 14-29), padding with the op identity.
    __shared__ Acc part[32];
    Acc w = T::warp(v);
    if (nw == 1) return T::to_grid(w);
    if (lane == 0) part[wid] = w;
    __syncthreads();
    Grid g = T::gident();
    if (wid == 0) {
      Acc x = lane < nw ? part[lane] : T::ident();
      g = T::to_grid(T::warp(x));
    }
    return g;
  } else if constexpr (BC == BC_ATOMIC_WARP || BC == BC_ATOMIC_ALL) {
    // "VA2+S" (Fig. 3(b) with the shuffle pass) or "VA1"
    // (Fig. 3(a)): one shared accumulator updated atomically by lane 0
    // of every warp, or by every thread.
    __shared__ Grid acc;
    if (threadIdx.x == 0) acc = T::gident();
    __syncthreads();
    if constexpr (BC == BC_ATOMIC_WARP) {
      Acc w = T::warp(v);
      if (lane == 0) T::gred(&acc, T::to_grid(w));
    } else {
      T::gred(&acc, T::to_grid(v));
    }
    __syncthreads();
    return acc;
  } else {
    // "V": shared tree, one barrier per step (Fig. 1(c) lines 9-13 with the
    // barrier Volta+ needs -- DESIGN.md reading R6).  blockDim.x must be a power of two.
    __shared__ Acc tmp[1024];
    tmp[threadIdx.x] = v;
    __syncthreads();
    for (int s = blockDim.x >> 1; s > 0; s >>= 1) {
      if ((int)threadIdx.x < s) tmp[threadIdx.x] = T::comb(tmp[threadIdx.x], tmp[threadIdx.x + s]);
      __syncthreads();
    }
    return T::to_grid(tmp[0]);
  }
}

// Fixed-order reduction of `count` Grid values by the whole block: thread t
// folds t, t+B, t+2B, ... then a warp butterfly, the warps' results meet in
// shared memory and warp 0 butterflies them (two barriers, deterministic).
// Reads with ld.global.cg (L2) since the values were written by other SMs.
template <class T>
__device__ __forceinline__ typename T::Grid reduce_grid_values(const typename T::Grid* vals, long long count) {
  using Grid = typename T::Grid;
  __shared__ Grid gpart[32];
  // 4 independent loads in flight per thread (values are L2-resident)
  Grid x0 = T::gident(), x1 = T::gident(), x2 = T::gident(), x3 = T::gident();
  const long long B = blockDim.x;
  long long i = threadIdx.x;
#pragma unroll 1
  for (; i + 3 * B < count; i += 4 * B) {
    const Grid v0 = __ldcg(vals + i), v1 = __ldcg(vals + i + B), v2 = __ldcg(vals + i + 2 * B), v3 = __ldcg(vals + i + 3 * B);
    x0 = T::gcomb(x0, v0);
    x1 = T::gcomb(x1, v1);
    x2 = T::gcomb(x2, v2);
    x3 = T::gcomb(x3, v3);
  }
#pragma unroll 1
  for (; i < count; i += B) x0 = T::gcomb(x0, __ldcg(vals + i));
  Grid x = T::gcomb(T::gcomb(x0, x1), T::gcomb(x2, x3));
  x = T::gwarp(x);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  __syncthreads();  // gpart may still be read by a previous use in this block
  if (lane == 0) gpart[wid] = x;
  __syncthreads();
  if (wid == 0) {
    Grid y = lane < nw ? gpart[lane] : T::gident();
    x = T::gwarp(y);
  }
  return x;  // valid in thread 0
}

}  // namespace rb
