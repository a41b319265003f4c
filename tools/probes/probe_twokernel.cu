// probe_twokernel.cu -- why does CUB's two-kernel DeviceReduce beat the
// library's TWO_PASS at 2-4 MB on B200?  Not product code.  Graph of R calls
// over cold regions, device time per call, all in one process:
//   cub            : cub::DeviceReduce::Sum (2 kernels, no PDL in CUDA 12.9)
//   lean2          : a minimal partials kernel (256 thr x 4 x 16 B, float
//                    partials) + a one-block final kernel, plain launches
//   lean2_pdl      : the same with programmatic stream serialisation (wait
//                    first, trigger after the loads)
//   lean2_v8       : 256 thr x 2 x 32 B loads (the library's 256-bit form)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_twokernel probe_twokernel.cu
#include <cub/device/device_reduce.cuh>
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

template <bool PDL, bool V8>
__global__ void __launch_bounds__(256) k_part(const float* __restrict__ in, float* partials) {
  if (PDL) asm volatile("griddepcontrol.wait;" ::: "memory");
  float acc = 0.f;
  if (V8) {
    const char* base = (const char*)in + ((size_t)blockIdx.x * 256 * 2 + threadIdx.x) * 32;
    uint32_t r[2][8];
#pragma unroll
    for (int u = 0; u < 2; ++u)
      asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]), "=r"(r[u][4]), "=r"(r[u][5]),
                     "=r"(r[u][6]), "=r"(r[u][7]) : "l"(base + (size_t)u * 256 * 32));
#pragma unroll
    for (int u = 0; u < 2; ++u)
#pragma unroll
      for (int k = 0; k < 8; ++k) acc += __uint_as_float(r[u][k]);
  } else {
    const float4* base = (const float4*)in + (size_t)blockIdx.x * 256 * 4 + threadIdx.x;
    float4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = __ldg(base + u * 256);
#pragma unroll
    for (int u = 0; u < 4; ++u) acc += (v[u].x + v[u].y) + (v[u].z + v[u].w);
  }
  if (PDL) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ float part[8];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x < 32) {
    float v = threadIdx.x < 8 ? part[threadIdx.x] : 0.f;
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (threadIdx.x == 0) partials[blockIdx.x] = v;
  }
}

template <bool PDL>
__global__ void __launch_bounds__(256) k_final(const float* partials, int count, float* out) {
  if (PDL) asm volatile("griddepcontrol.wait;" ::: "memory");
  float x = 0.f;
  for (int i = threadIdx.x; i < count; i += 256) x += partials[i];
  for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  __shared__ float part[8];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = x;
  __syncthreads();
  if (threadIdx.x < 32) {
    float v = threadIdx.x < 8 ? part[threadIdx.x] : 0.f;
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (threadIdx.x == 0) *out = v;
  }
}

template <class K, class... A>
void launch(bool pdl, K kern, int grid, cudaStream_t s, A... a) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(256);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  CK(cudaLaunchKernelEx(&cfg, kern, a...));
}

int main() {
  const size_t pool_bytes = 1ull << 30;
  float* pool;
  CK(cudaMalloc(&pool, pool_bytes));
  CK(cudaMemset(pool, 0, pool_bytes));
  float *partials, *out;
  CK(cudaMalloc(&partials, 1 << 20));
  CK(cudaMalloc(&out, 4096 * 4));
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
  CK(cub::DeviceReduce::Sum(tmp, tmp_bytes, pool, out, 1 << 23));
  CK(cudaMalloc(&tmp, tmp_bytes));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  const char* names[] = {"cub", "lean2", "lean2_pdl", "lean2_v8", "lean2_v8_pdl"};
  for (int lb = 19; lb <= 23; ++lb) {
    const size_t n = 1ull << lb;
    const int grid = (int)(n / 4096);  // 256 threads x 16 floats
    const int R = 100;
    const int fit = (int)(pool_bytes / (n * 4));
    for (int v = 0; v < 5; ++v) {
      float best = 1e30f;
      for (int rep = 0; rep < 3; ++rep) {
        cudaGraphExec_t ge[2];
        for (int gi = 0; gi < 2; ++gi) {
          cudaGraph_t g;
          CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
          for (int i = 0; i < R; ++i) {
            const float* in = pool + (size_t)((gi * R + i) % fit) * n;
            float* o = out + (i % 4096);
            if (v == 0) {
              CK(cub::DeviceReduce::Sum(tmp, tmp_bytes, in, o, (int)n, s));
            } else {
              const bool pdl = v == 2 || v == 4;
              if (v <= 2) launch(pdl, k_part<true, false>, grid, s, in, partials);
              else launch(pdl, k_part<true, true>, grid, s, in, partials);
              launch(pdl, k_final<true>, 1, s, (const float*)partials, grid, o);
            }
          }
          CK(cudaStreamEndCapture(s, &g));
          CK(cudaGraphInstantiate(&ge[gi], g, 0));
          cudaGraphDestroy(g);
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
        cudaGraphExecDestroy(ge[0]);
        cudaGraphExecDestroy(ge[1]);
      }
      printf("n=2^%d %-14s %8.3f us\n", lb, names[v], best);
    }
  }
  return 0;
}
