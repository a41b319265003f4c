// probe_mid.cu -- where does a medium-size (1-64 MB) reduction's time go on
// B200?  Not product code.  Graph of R back-to-back calls over cold regions,
// every kernel launched with programmatic stream serialisation, device time per
// call.  Variants of one 256-thread x U=4 x 32 B tile-per-block streaming
// kernel (fp32 sum):
//   store   : each block stores its partial to partials[blockIdx] (no combine;
//             the single-kernel floor)
//   atomic  : + red.global.add.f64 into one of 32 slots + acq_rel ticket; the
//             last block exchanges the slots and writes the result (the
//             library's "DT,A")
//   *_early : the same with the first tile loaded before griddepcontrol.wait
//   *_trig0 : every block triggers its dependents at its start (instead of
//             after its loads)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_mid probe_mid.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

struct P {
  const char* in;
  double* partials;
  double* slots;
  unsigned* ticket;
  float* out;
  long long tiles;
  unsigned epoch;
};

__device__ __forceinline__ void ldv8(const void* p, uint32_t (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
               : "l"(p));
}

// EARLY: 0 none, 1 first tile into registers before the wait, 2 bulk L2
// prefetch of every tile this CTA will read before the wait.  The grid may be
// smaller than the tile count (persistent: CTA b reads tiles b, b+G, ...).
template <int MODE, int EARLY, bool TRIG0>  // MODE 0 store, 1 atomic, 2 relaxed ticket, 3 packed, 4 flags,
                                            // 5 flags polled by the fixed block G-1 (no ticket)
__global__ void __launch_bounds__(256) k(P p) {
  const long long tiles = p.tiles;
  uint32_t r[4][8];
  if (EARLY == 1) {
    const char* base = p.in + ((size_t)blockIdx.x * 256 * 4 + threadIdx.x) * 32;
#pragma unroll
    for (int u = 0; u < 4; ++u) ldv8(base + (size_t)u * 256 * 32, r[u]);
  }
  if (EARLY == 2 && threadIdx.x == 0) {
    for (long long t = blockIdx.x; t < tiles; t += gridDim.x)
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p.in + (size_t)t * 32768), "r"(32768) : "memory");
  }
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (TRIG0) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  float acc = 0.f;
  long long t = blockIdx.x;
  if (EARLY == 1) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      float x = ((__uint_as_float(r[u][0]) + __uint_as_float(r[u][1])) + (__uint_as_float(r[u][2]) + __uint_as_float(r[u][3]))) +
                ((__uint_as_float(r[u][4]) + __uint_as_float(r[u][5])) + (__uint_as_float(r[u][6]) + __uint_as_float(r[u][7])));
      acc += x;
    }
    t += gridDim.x;
  }
#pragma unroll 1
  for (; t < tiles; t += gridDim.x) {
    const char* base = p.in + ((size_t)t * 256 * 4 + threadIdx.x) * 32;
#pragma unroll
    for (int u = 0; u < 4; ++u) ldv8(base + (size_t)u * 256 * 32, r[u]);
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      float x = ((__uint_as_float(r[u][0]) + __uint_as_float(r[u][1])) + (__uint_as_float(r[u][2]) + __uint_as_float(r[u][3]))) +
                ((__uint_as_float(r[u][4]) + __uint_as_float(r[u][5])) + (__uint_as_float(r[u][6]) + __uint_as_float(r[u][7])));
      acc += x;
    }
  }
  if (!TRIG0) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ float part[8];
  __shared__ int last;
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x < 32) {
    float v = threadIdx.x < 8 ? part[threadIdx.x] : 0.f;
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (threadIdx.x == 0) {
      if (MODE == 0) {
        p.partials[blockIdx.x] = (double)v;
      } else if (MODE == 1 || MODE == 2) {
        atomicAdd(p.slots + (blockIdx.x & 31) * 32, (double)v);
        unsigned old;
        if (MODE == 1) asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(old) : "l"(p.ticket) : "memory");
        else asm volatile("atom.add.relaxed.gpu.global.u32 %0, [%1], 1;" : "=r"(old) : "l"(p.ticket) : "memory");
        last = old == gridDim.x - 1;
      } else if (MODE == 3) {
        // int32-style packed word: count at bit 48, sum mod 2^32 in bits 0-31
        const unsigned long long add = (1ull << 48) | (unsigned long long)(unsigned)__float_as_uint(v);
        unsigned long long old = atomicAdd((unsigned long long*)p.slots, add);
        last = (unsigned)(old >> 48) == gridDim.x - 1;
        if (last) {
          *p.out = __uint_as_float((unsigned)(old + add));
          atomicExch((unsigned long long*)p.slots, 0ull);
        }
      } else if (MODE == 5) {
        if (blockIdx.x != gridDim.x - 1) {
          const unsigned long long b = (unsigned long long)__double_as_longlong((double)v);
          asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1, %2, %3, %4};" :: "l"(p.partials + 2 * blockIdx.x),
                       "r"((unsigned)b), "r"(p.epoch), "r"((unsigned)(b >> 32)), "r"(p.epoch) : "memory");
        }
        last = blockIdx.x == gridDim.x - 1;
        part[0] = v;
      } else {
        // flag-in-data partial {value bits, epoch} then a relaxed ticket
        const unsigned epoch = p.epoch;
        const unsigned long long b = (unsigned long long)__double_as_longlong((double)v);
        asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1, %2, %3, %4};" :: "l"(p.partials + 2 * blockIdx.x),
                     "r"((unsigned)b), "r"(epoch), "r"((unsigned)(b >> 32)), "r"(epoch) : "memory");
        unsigned old;
        asm volatile("atom.add.relaxed.gpu.global.u32 %0, [%1], 1;" : "=r"(old) : "l"(p.ticket) : "memory");
        last = old == gridDim.x - 1;
      }
    }
  }
  if (MODE == 1 || MODE == 2) {
    __syncthreads();
    if (last && threadIdx.x < 32) {
      unsigned long long b = atomicExch((unsigned long long*)(p.slots + threadIdx.x * 32), 0ull);
      double x = __longlong_as_double((long long)b);
      for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
      if (threadIdx.x == 0) {
        *p.out = (float)x;
        atomicExch(p.ticket, 0u);
      }
    }
  }
  if (MODE == 5) {
    __syncthreads();
    if (last) {
      double x = threadIdx.x == 0 ? (double)part[0] : 0.0;
      const int G1 = (int)gridDim.x - 1;
      for (int i0 = threadIdx.x; i0 < G1; i0 += 256 * 8) {
        unsigned a[8], fa[8], b2[8], fb[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          fa[j] = fb[j] = p.epoch; a[j] = b2[j] = 0u;
          if (i0 + 256 * j < G1)
            asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(a[j]), "=r"(fa[j]), "=r"(b2[j]), "=r"(fb[j])
                         : "l"(p.partials + 2 * (i0 + 256 * j)) : "memory");
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          while (fa[j] != p.epoch || fb[j] != p.epoch) {
            __nanosleep(20);
            asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(a[j]), "=r"(fa[j]), "=r"(b2[j]), "=r"(fb[j])
                         : "l"(p.partials + 2 * (i0 + 256 * j)) : "memory");
          }
          x += __longlong_as_double((long long)(((unsigned long long)b2[j] << 32) | a[j]));
        }
      }
      for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
      __shared__ double dp[8];
      __syncthreads();
      if ((threadIdx.x & 31) == 0) dp[threadIdx.x >> 5] = x;
      __syncthreads();
      if (threadIdx.x < 32) {
        double y = threadIdx.x < 8 ? dp[threadIdx.x] : 0.0;
        for (int o = 4; o; o >>= 1) y += __shfl_xor_sync(0xffffffffu, y, o);
        if (threadIdx.x == 0) *p.out = (float)y;
      }
    }
  }
  if (MODE == 4) {
    __syncthreads();
    if (last) {
      double x = 0.0;
      for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) {
        unsigned a, fa, b2, fb;
        do {
          asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(a), "=r"(fa), "=r"(b2), "=r"(fb)
                       : "l"(p.partials + 2 * i) : "memory");
        } while (fa != p.epoch || fb != p.epoch);
        x += __longlong_as_double((long long)(((unsigned long long)b2 << 32) | a));
      }
      for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
      if ((threadIdx.x & 31) == 0) atomicAdd(p.slots + 64, x);  // (timing probe: crude block sum)
      if (threadIdx.x == 0) {
        *p.out = (float)x;
        atomicExch(p.ticket, 0u);
      }
    }
  }
}

template <class F>
void launch(F kern, int grid, cudaStream_t s, P p) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(256);
  cfg.stream = s;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  a[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = a;
  cfg.numAttrs = 1;
  CK(cudaLaunchKernelEx(&cfg, kern, p));
}

typedef void (*KF)(P);

int main() {
  const size_t pool_bytes = 2ull << 30;
  char* pool;
  CK(cudaMalloc(&pool, pool_bytes));
  CK(cudaMemset(pool, 0, pool_bytes));
  double *partials, *slots;
  unsigned* ticket;
  float* out;
  CK(cudaMalloc(&partials, 1 << 24));
  CK(cudaMalloc(&slots, 32 * 32 * 8));
  CK(cudaMemset(slots, 0, 32 * 32 * 8));
  CK(cudaMalloc(&ticket, 4));
  CK(cudaMemset(ticket, 0, 4));
  CK(cudaMalloc(&out, 4096 * 4));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  struct V { const char* name; KF f; int per_sm; };  // per_sm 0: one tile per CTA
  V vs[] = {{"store_pf", k<0, 2, false>, 0}, {"atomic_pf", k<1, 2, false>, 0}, {"packed_int_pf", k<3, 2, false>, 0},
            {"flags_fixed_pf", k<5, 2, false>, 0}, {"flags_fixed", k<5, 0, false>, 0}, {"flags_fixed_early", k<5, 1, false>, 0},
            {"atomic_early", k<1, 1, false>, 0}};
  V vs_old[] = {{"store", k<0, 0, false>, 0}, {"atomic", k<1, 0, false>, 0}, {"atomic_relaxed_WRONG", k<2, 0, false>, 0},
            {"packed_int", k<3, 0, false>, 0}, {"flags_relaxed", k<4, 0, false>, 0},
            {"store_pf", k<0, 2, false>, 0}, {"atomic_pf", k<1, 2, false>, 0}, {"packed_int_pf", k<3, 2, false>, 0},
            {"flags_pf", k<4, 2, false>, 0}, {"atomic_early", k<1, 1, false>, 0}, {"packed_early", k<3, 1, false>, 0},
            {"flags_early", k<4, 1, false>, 0}};
  for (int lb = 20; lb <= 28; lb += 2) {
    (void)vs_old;
    const size_t bytes = 1ull << lb;
    const long long tiles = (long long)(bytes / (256 * 4 * 32));
    const int R = 100;
    const size_t stride = bytes;
    const int fit = (int)(pool_bytes / stride);
    for (const V& v : vs) {
      const int grid = v.per_sm == 0 ? (int)tiles : (int)(tiles < 148ll * v.per_sm ? tiles : 148ll * v.per_sm);
      float best = 1e30f;
      for (int rep = 0; rep < 3; ++rep) {
        cudaGraph_t g[2];
        cudaGraphExec_t ge[2];
        for (int gi = 0; gi < 2; ++gi) {
          CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
          for (int i = 0; i < R; ++i) {
            const int reg = (gi * R + i) % fit;
            P p{pool + (size_t)reg * stride, partials, slots, ticket, out + (i % 4096), tiles, (unsigned)(rep * 1000 + gi * 200 + i + 1)};
            launch(v.f, grid, s, p);
          }
          CK(cudaStreamEndCapture(s, &g[gi]));
          CK(cudaGraphInstantiate(&ge[gi], g[gi], 0));
        }
        cudaEvent_t a, b;
        CK(cudaEventCreate(&a));
        CK(cudaEventCreate(&b));
        CK(cudaGraphLaunch(ge[0], s));
        CK(cudaEventRecord(a, s));
        CK(cudaGraphLaunch(ge[1], s));
        CK(cudaEventRecord(b, s));
        CK(cudaEventSynchronize(b));
        float ms;
        CK(cudaEventElapsedTime(&ms, a, b));
        best = ms * 1e3f / R < best ? ms * 1e3f / R : best;
        for (int gi = 0; gi < 2; ++gi) {
          cudaGraphExecDestroy(ge[gi]);
          cudaGraphDestroy(g[gi]);
        }
      }
      printf("bytes=2^%d grid=%6d %-24s %8.3f us  %7.1f GB/s\n", lb, grid, v.name, best, bytes / (best * 1e3));
    }
  }
  return 0;
}
