// Throwaway probe (not product code): what makes CUB's two-kernel reduce faster
// than ours at 1M-16M fp32 elements?  Graph-timed (100 calls, cold regions):
//   cub      : cub::DeviceReduce::Sum
//   lean     : 256 thr x 2 x 32 B tiles, tree fold, warp shfl + smem block
//              reduce, partial store; + a 256-thread partials kernel
//   lean+pdl : the same launched with programmatic stream serialisation
//              (griddepcontrol.wait / launch_dependents)
#include <cub/device/device_reduce.cuh>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

template <bool PDL, int U>
__global__ void __launch_bounds__(256) k_main(const float* __restrict__ in, double* partials) {
  if (PDL) asm volatile("griddepcontrol.wait;" ::: "memory");
  const char* base = (const char*)in + ((size_t)blockIdx.x * 256 * U + threadIdx.x) * 32;
  uint32_t r[U][8];
#pragma unroll
  for (int u = 0; u < U; ++u)
    asm("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]), "=r"(r[u][4]), "=r"(r[u][5]), "=r"(r[u][6]), "=r"(r[u][7])
        : "l"(base + (size_t)u * 256 * 32));
  float acc = 0.f;
#pragma unroll
  for (int u = 0; u < U; ++u) {
    float t = ((__uint_as_float(r[u][0]) + __uint_as_float(r[u][1])) + (__uint_as_float(r[u][2]) + __uint_as_float(r[u][3]))) +
              ((__uint_as_float(r[u][4]) + __uint_as_float(r[u][5])) + (__uint_as_float(r[u][6]) + __uint_as_float(r[u][7])));
    acc += t;
  }
  if (PDL) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ float part[8];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x < 32) {
    float v = threadIdx.x < 8 ? part[threadIdx.x] : 0.f;
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (threadIdx.x == 0) partials[blockIdx.x] = (double)v;
  }
}

template <bool PDL>
__global__ void __launch_bounds__(256) k_final(const double* partials, int count, float* out) {
  if (PDL) asm volatile("griddepcontrol.wait;" ::: "memory");
  double x = 0;
  for (int i = threadIdx.x; i < count; i += 256) x += partials[i];
  for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  __shared__ double part[8];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = x;
  __syncthreads();
  if (threadIdx.x < 32) {
    double v = threadIdx.x < 8 ? part[threadIdx.x] : 0.0;
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (threadIdx.x == 0) *out = (float)v;
  }
}

template <class K, class... A>
static void launch(bool pdl, K kern, int grid, int block, cudaStream_t s, A... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  CK(cudaLaunchKernelEx(&cfg, kern, args...));
}

int main() {
  const size_t pool_bytes = (size_t)2 << 30;
  float* pool; CK(cudaMalloc(&pool, pool_bytes)); CK(cudaMemset(pool, 0, pool_bytes));
  double* partials; CK(cudaMalloc(&partials, 1 << 24));
  float* out; CK(cudaMalloc(&out, 4096 * 4));
  void* tmp = nullptr; size_t tmp_bytes = 0;
  cub::DeviceReduce::Sum(nullptr, tmp_bytes, pool, out, 1 << 28);
  CK(cudaMalloc(&tmp, tmp_bytes));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (size_t n : {(size_t)1 << 18, (size_t)1 << 20, (size_t)1 << 22, (size_t)1 << 24, (size_t)1 << 26}) {
    const size_t bytes = n * 4;
    const int R = (int)std::max<size_t>(5, std::min<size_t>(100, (size_t)(400 << 20) / bytes));
    const size_t nreg = pool_bytes / bytes;
    for (int variant = 0; variant < 5; ++variant) {
      auto one = [&](int r) {
        const float* in = pool + (size_t)(r % nreg) * n;
        if (variant == 0) {
          size_t tb = tmp_bytes;
          cub::DeviceReduce::Sum(tmp, tb, in, out + (r % 4096), (int64_t)n, s);
        } else {
          const bool pdl = variant == 2 || variant == 4;
          const int U = variant <= 2 ? 2 : 4;
          const int grid = (int)(n / (256 * 8 * U));
          if (U == 2) launch(pdl, k_main<true, 2>, grid, 256, s, in, partials);
          else launch(pdl, k_main<true, 4>, grid, 256, s, in, partials);
          launch(pdl, k_final<true>, 1, 256, s, (const double*)partials, grid, out + (r % 4096));
        }
      };
      float best = 1e9;
      for (int rep = 0; rep < 3; ++rep) {
        cudaGraph_t g; cudaGraphExec_t ge;
        CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
        for (int r = 0; r < R; ++r) one(rep * R + r);
        CK(cudaStreamEndCapture(s, &g));
        CK(cudaGraphInstantiate(&ge, g, 0));
        CK(cudaGraphLaunch(ge, s));
        cudaEventRecord(e0, s);
        CK(cudaGraphLaunch(ge, s));
        cudaEventRecord(e1, s);
        CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        best = std::min(best, ms * 1e3f / R);
        cudaGraphExecDestroy(ge); cudaGraphDestroy(g);
      }
      const char* names[] = {"cub", "lean U2", "lean U2 pdl", "lean U4", "lean U4 pdl"};
      printf("n=%9zu %-12s %8.3f us\n", n, names[variant], best);
    }
  }
  return 0;
}
