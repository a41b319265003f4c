// Throwaway probe (not product code): does staging tiles through shared memory
// with TMA bulk copies (cp.async.bulk + mbarrier) or cp.async raise the bytes in
// flight per SM -- and so the HBM read throughput -- over register-staged
// 256-bit LDG, for an fp32 sum with the same atomic grid combine?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o probe_bulk probe_bulk.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ float warp_sum(float v) {
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
// block sum -> thread 0; then atomic grid combine with ticket (same as product GC_ATOMIC, 1 slot)
__device__ __forceinline__ void finish(float v, double* acc, unsigned* ticket, float* out) {
  __shared__ float part[32];
  __shared__ int last;
  v = warp_sum(v);
  int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (lane == 0) part[w] = v;
  __syncthreads();
  if (w == 0) {
    v = lane < nw ? part[lane] : 0.f;
    v = warp_sum(v);
    if (lane == 0) {
      atomicAdd(acc, (double)v);
      __threadfence();
      unsigned t = atomicAdd(ticket, 1u);
      last = (t == gridDim.x - 1);
      if (last) {
        __threadfence();
        double s = atomicExch((unsigned long long*)acc, 0ull);
        *out = (float)__longlong_as_double(s);
        *ticket = 0;
      }
    }
  }
}

// (a) register-staged 256-bit loads (product kernel's S2)
template <int U>
__global__ void __launch_bounds__(1024) k_ldg(const float* in, size_t nvec, double* acc, unsigned* ticket, float* out) {
  const char* base = (const char*)in;
  size_t v0 = (size_t)blockIdx.x * blockDim.x * U + threadIdx.x;
  float a[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  uint32_t r[U][8];
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const char* p = base + (v0 + (size_t)u * blockDim.x) * 32;
    asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]), "=r"(r[u][4]), "=r"(r[u][5]),
                   "=r"(r[u][6]), "=r"(r[u][7]) : "l"(p));
  }
#pragma unroll
  for (int u = 0; u < U; ++u)
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] += __uint_as_float(r[u][k]);
  float v = ((a[0] + a[1]) + (a[2] + a[3])) + ((a[4] + a[5]) + (a[6] + a[7]));
  finish(v, acc, ticket, out);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// (b) one TMA bulk copy of the whole tile per block (tile = TB bytes), then an smem reduce.
// (c) the same, but the tile is split into S bulk copies on S mbarriers so the
//     reduce of piece s overlaps the arrival of the later pieces.
template <int S>
__global__ void __launch_bounds__(1024) k_bulk(const float* in, int tile_bytes, double* acc, unsigned* ticket, float* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ __align__(8) uint64_t mbar[S];
  const int piece = tile_bytes / S;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&mbar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const char* src = (const char*)in + (size_t)blockIdx.x * tile_bytes;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(&mbar[s])), "r"(piece) : "memory");
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   :: "r"(smem_u32(sm + s * piece)), "l"(src + (size_t)s * piece), "r"(piece), "r"(smem_u32(&mbar[s]))
                   : "memory");
    }
  }
  float a[4] = {0, 0, 0, 0};
  for (int s = 0; s < S; ++s) {
    uint32_t done = 0;
    while (!done)
      asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                   : "=r"(done) : "r"(smem_u32(&mbar[s])) : "memory");
    const float4* q = (const float4*)(sm + s * piece);
    for (int i = threadIdx.x; i < piece / 16; i += blockDim.x) {
      float4 x = q[i];
      a[0] += x.x; a[1] += x.y; a[2] += x.z; a[3] += x.w;
    }
  }
  finish((a[0] + a[1]) + (a[2] + a[3]), acc, ticket, out);
}

// (d) cp.async (LDGSTS) 16 B per instruction, U per thread, then smem reduce
template <int U>
__global__ void __launch_bounds__(1024) k_cpasync(const float* in, double* acc, unsigned* ticket, float* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  const int tile = blockDim.x * U * 16;
  const char* src = (const char*)in + (size_t)blockIdx.x * tile;
#pragma unroll
  for (int u = 0; u < U; ++u) {
    int off = (u * blockDim.x + threadIdx.x) * 16;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(smem_u32(sm + off)), "l"(src + off) : "memory");
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
  float a[4] = {0, 0, 0, 0};
#pragma unroll
  for (int u = 0; u < U; ++u) {
    float4 x = *(const float4*)(sm + (u * blockDim.x + threadIdx.x) * 16);  // own data: no barrier needed
    a[0] += x.x; a[1] += x.y; a[2] += x.z; a[3] += x.w;
  }
  finish((a[0] + a[1]) + (a[2] + a[3]), acc, ticket, out);
}

int main() {
  const size_t bytes = (size_t)2 << 30;  // 2 GiB pool; each config reads 1 GiB at offset alternating
  float* buf; CK(cudaMalloc(&buf, bytes));
  CK(cudaMemset(buf, 0, bytes));
  double* acc; unsigned* ticket; float* out;
  CK(cudaMalloc(&acc, 8)); CK(cudaMalloc(&ticket, 4)); CK(cudaMalloc(&out, 4));
  CK(cudaMemset(acc, 0, 8)); CK(cudaMemset(ticket, 0, 4));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const size_t n1 = (size_t)1 << 30;  // bytes per call
  auto run = [&](const char* name, auto launch) {
    for (int w = 0; w < 3; ++w) launch(w & 1);
    cudaEventRecord(e0);
    const int R = 20;
    for (int r = 0; r < R; ++r) launch(r & 1);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    cudaError_t e = cudaGetLastError();
    printf("%-40s %8.2f us  %8.1f GB/s %s\n", name, ms * 1e3 / R, n1 / (ms * 1e-3 / R) / 1e9, e == cudaSuccess ? "" : cudaGetErrorString(e));
  };
  char name[128];
  for (int B : {128, 256, 512}) {
    sprintf(name, "ldg U4 B%d", B);
    run(name, [&](int h) { k_ldg<4><<<n1 / (B * 4 * 32), B>>>(buf + h * (n1 / 4), 0, acc, ticket, out); });
    sprintf(name, "ldg U8 B%d", B);
    if (B <= 512) run(name, [&](int h) { k_ldg<8><<<n1 / (B * 8 * 32), B>>>(buf + h * (n1 / 4), 0, acc, ticket, out); });
  }
  for (int tile : {16384, 32768, 65536}) {
    for (int B : {128, 256, 512}) {
      cudaFuncSetAttribute(k_bulk<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      cudaFuncSetAttribute(k_bulk<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      cudaFuncSetAttribute(k_bulk<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      sprintf(name, "bulk S1 tile%dK B%d", tile / 1024, B);
      run(name, [&](int h) { k_bulk<1><<<n1 / tile, B, tile>>>(buf + h * (n1 / 4), tile, acc, ticket, out); });
      sprintf(name, "bulk S2 tile%dK B%d", tile / 1024, B);
      run(name, [&](int h) { k_bulk<2><<<n1 / tile, B, tile>>>(buf + h * (n1 / 4), tile, acc, ticket, out); });
      sprintf(name, "bulk S4 tile%dK B%d", tile / 1024, B);
      run(name, [&](int h) { k_bulk<4><<<n1 / tile, B, tile>>>(buf + h * (n1 / 4), tile, acc, ticket, out); });
    }
  }
  for (int B : {128, 256, 512}) {
    cudaFuncSetAttribute(k_cpasync<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(k_cpasync<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    sprintf(name, "cp.async U8 B%d", B);
    run(name, [&](int h) { k_cpasync<8><<<n1 / (B * 8 * 16), B, B * 8 * 16>>>(buf + h * (n1 / 4), acc, ticket, out); });
    sprintf(name, "cp.async U16 B%d", B);
    run(name, [&](int h) { k_cpasync<16><<<n1 / (B * 16 * 16), B, B * 16 * 16>>>(buf + h * (n1 / 4), acc, ticket, out); });
  }
  float h; cudaMemcpy(&h, out, 4, cudaMemcpyDeviceToHost);
  printf("out %f (expect 0)\n", h);
  return 0;
}
