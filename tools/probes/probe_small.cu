// Throwaway probe (not product code): why is CUB's DeviceReduceKernel faster
// than ours at 4-64 MB?  Compare load flavours (256-bit vs 128-bit, .nc with
// and without L1::no_allocate, plain) for a one-tile-per-block partial sum
// (16 KB tiles, 256 threads, 64 B per thread), cold inputs (rotating buffers),
// device time per launch from events around 40 back-to-back launches.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int KIND>  // 0: v8 nc na, 1: v4 nc na, 2: v4 nc, 3: v4 plain, 4: v8 nc (no na)
__global__ void __launch_bounds__(256) k_part(const float* in, float* partials) {
  const char* base = (const char*)in + (size_t)blockIdx.x * 16384;
  float a[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  if (KIND == 0 || KIND == 4) {
    uint32_t r[2][8];
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const char* p = base + (u * 256 + threadIdx.x) * 32;
      if (KIND == 0)
        asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]), "=r"(r[u][4]), "=r"(r[u][5]), "=r"(r[u][6]), "=r"(r[u][7]) : "l"(p));
      else
        asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]), "=r"(r[u][4]), "=r"(r[u][5]), "=r"(r[u][6]), "=r"(r[u][7]) : "l"(p));
    }
#pragma unroll
    for (int u = 0; u < 2; ++u)
#pragma unroll
      for (int k = 0; k < 8; ++k) a[k] += __uint_as_float(r[u][k]);
  } else {
    uint32_t r[4][4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const char* p = base + (u * 256 + threadIdx.x) * 16;
      if (KIND == 1)
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]) : "l"(p));
      else if (KIND == 2)
        asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]) : "l"(p));
      else
        asm volatile("ld.global.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]) : "l"(p));
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
      for (int k = 0; k < 4; ++k) a[k] += __uint_as_float(r[u][k]);
  }
  float v = ((a[0] + a[1]) + (a[2] + a[3])) + ((a[4] + a[5]) + (a[6] + a[7]));
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  __shared__ float part[8];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = v;
  __syncthreads();
  if (threadIdx.x < 32) {
    v = threadIdx.x < 8 ? part[threadIdx.x] : 0.f;
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (threadIdx.x == 0) partials[blockIdx.x] = v;
  }
}

int main() {
  const size_t pool = (size_t)4 << 30;
  float* buf; cudaMalloc(&buf, pool); cudaMemset(buf, 0, pool);
  float* part; cudaMalloc(&part, 1 << 24);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[] = {"v8 nc na", "v4 nc na", "v4 nc", "v4 plain", "v8 nc"};
  for (size_t bytes : {(size_t)1 << 22, (size_t)1 << 24, (size_t)1 << 26}) {
    const int grid = (int)(bytes / 16384);
    const int R = 40;
    for (int kind = 0; kind < 5; ++kind) {
      auto launch = [&](int r) {
        const float* in = (const float*)((const char*)buf + ((size_t)r * bytes) % (pool - bytes));
        switch (kind) {
          case 0: k_part<0><<<grid, 256>>>(in, part); break;
          case 1: k_part<1><<<grid, 256>>>(in, part); break;
          case 2: k_part<2><<<grid, 256>>>(in, part); break;
          case 3: k_part<3><<<grid, 256>>>(in, part); break;
          case 4: k_part<4><<<grid, 256>>>(in, part); break;
        }
      };
      for (int r = 0; r < 3; ++r) launch(r);
      cudaEventRecord(e0);
      for (int r = 0; r < R; ++r) launch(r + 7);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      printf("%9zu B  %-10s %8.2f us/launch %8.1f GB/s\n", bytes, names[kind], ms * 1e3 / R, bytes / (ms * 1e-3 / R) / 1e9);
    }
  }
  return 0;
}
