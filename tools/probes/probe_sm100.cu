// Throwaway hardware probe (not product code): fp min/max signed-zero / NaN
// semantics of the sm_100a min/max instructions, and a read-bandwidth sweep of
// simple grid-stride streaming loops, to ground the kernel design in DESIGN.md.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe probe_sm100.cu
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); return 1; } } while (0)

__device__ __forceinline__ float max_nan(float a, float b) {
  float r; asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float min_nan(float a, float b) {
  float r; asm("min.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float max_plain(float a, float b) {
  float r; asm("max.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float min_plain(float a, float b) {
  float r; asm("min.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ double max_d(double a, double b) {
  double r; asm("max.f64 %0, %1, %2;" : "=d"(r) : "d"(a), "d"(b)); return r; }
__device__ __forceinline__ double min_d(double a, double b) {
  double r; asm("min.f64 %0, %1, %2;" : "=d"(r) : "d"(a), "d"(b)); return r; }
__device__ __forceinline__ float redux_max_nan(float a) {
  float r; asm("redux.sync.max.NaN.f32 %0, %1, 0xffffffff;" : "=f"(r) : "f"(a)); return r; }
__device__ __forceinline__ float redux_min_nan(float a) {
  float r; asm("redux.sync.min.NaN.f32 %0, %1, 0xffffffff;" : "=f"(r) : "f"(a)); return r; }

__global__ void k_sem(const float* a, const float* b, int npairs, uint32_t* out) {
  int i = threadIdx.x;
  if (i < npairs) {
    out[i * 6 + 0] = __float_as_uint(max_nan(a[i], b[i]));
    out[i * 6 + 1] = __float_as_uint(min_nan(a[i], b[i]));
    out[i * 6 + 2] = __float_as_uint(max_plain(a[i], b[i]));
    out[i * 6 + 3] = __float_as_uint(min_plain(a[i], b[i]));
    double da = a[i], db = b[i];
    unsigned long long mx = __double_as_longlong(max_d(da, db));
    unsigned long long mn = __double_as_longlong(min_d(da, db));
    out[i * 6 + 4] = (uint32_t)(mx >> 32);
    out[i * 6 + 5] = (uint32_t)(mn >> 32);
  }
}

__global__ void k_redux(const float* v, uint32_t* out) {
  float x = v[threadIdx.x];
  float mx = redux_max_nan(x), mn = redux_min_nan(x);
  if (threadIdx.x == 0) { out[0] = __float_as_uint(mx); out[1] = __float_as_uint(mn); }
}

// ---- bandwidth probes -------------------------------------------------------
__device__ __forceinline__ void ld8(const void* p, uint32_t (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
      : "l"(p));
}
__device__ __forceinline__ void ld4(const void* p, uint32_t (&r)[4]) {
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "l"(p));
}

template <int VB, int U>  // VB = bytes per vector (16/32), U = unroll
__global__ void k_bw(const float* __restrict__ in, size_t nvec, float* out) {
  const char* base = (const char*)in;
  size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  size_t i = tid;
  for (; i + (U - 1) * stride < nvec; i += U * stride) {
    if (VB == 32) {
      uint32_t r[U][8];
#pragma unroll
      for (int u = 0; u < U; ++u) ld8(base + (i + u * stride) * 32, r[u]);
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int k = 0; k < 8; ++k) acc[k] += __uint_as_float(r[u][k]);
    } else {
      uint32_t r[U][4];
#pragma unroll
      for (int u = 0; u < U; ++u) ld4(base + (i + u * stride) * 16, r[u]);
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[k] += __uint_as_float(r[u][k]);
    }
  }
  for (; i < nvec; i += stride) {
    if (VB == 32) { uint32_t r[8]; ld8(base + i * 32, r); for (int k = 0; k < 8; ++k) acc[k] += __uint_as_float(r[k]); }
    else { uint32_t r[4]; ld4(base + i * 16, r); for (int k = 0; k < 4; ++k) acc[k] += __uint_as_float(r[k]); }
  }
  float s = 0; for (int k = 0; k < 8; ++k) s += acc[k];
  if (s == 123456.0f) out[0] = s;  // keep the loads alive
}

// block-chunked (tile per block, stride across threads) variant
template <int U>
__global__ void k_bw_tile(const float* __restrict__ in, size_t nvec, float* out) {
  const char* base = (const char*)in;
  size_t per = (nvec + gridDim.x - 1) / gridDim.x;
  size_t beg = blockIdx.x * per, end = beg + per < nvec ? beg + per : nvec;
  float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  size_t i = beg + threadIdx.x;
  for (; i + (U - 1) * blockDim.x < end; i += U * blockDim.x) {
    uint32_t r[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) ld8(base + (i + u * blockDim.x) * 32, r[u]);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int k = 0; k < 8; ++k) acc[k] += __uint_as_float(r[u][k]);
  }
  for (; i < end; i += blockDim.x) { uint32_t r[8]; ld8(base + i * 32, r); for (int k = 0; k < 8; ++k) acc[k] += __uint_as_float(r[k]); }
  float s = 0; for (int k = 0; k < 8; ++k) s += acc[k];
  if (s == 123456.0f) out[0] = s;
}

template <typename K>
float time_kernel(K kern, int grid, int block, const float* in, size_t nvec, float* out, int reps) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int w = 0; w < 3; ++w) kern<<<grid, block>>>(in, nvec, out);
  cudaEventRecord(e0);
  for (int r = 0; r < reps; ++r) kern<<<grid, block>>>(in, nvec, out);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0); cudaEventDestroy(e1);
  return ms / reps;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  printf("device %s SMs %d L2 %d MB smem/SM %zu clock %d kHz memclk %d kHz bus %d\n", p.name,
         p.multiProcessorCount, p.l2CacheSize >> 20, p.sharedMemPerMultiprocessor, p.clockRate,
         p.memoryClockRate, p.memoryBusWidth);
  // ---- semantics
  const float nan_p = __builtin_nanf(""), ninf = -__builtin_inff();
  uint32_t negnan_bits = 0xFFC00001u; float nan_n; memcpy(&nan_n, &negnan_bits, 4);
  float ha[] = {-0.0f, 0.0f, 1.0f, nan_p, nan_n, -1.0f, ninf};
  float hb[] = {0.0f, -0.0f, nan_p, 1.0f, -1.0f, nan_n, -0.0f};
  int np = 7;
  float *da, *db; uint32_t* dout;
  CK(cudaMalloc(&da, 256)); CK(cudaMalloc(&db, 256)); CK(cudaMalloc(&dout, 1024));
  CK(cudaMemcpy(da, ha, np * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(db, hb, np * 4, cudaMemcpyHostToDevice));
  k_sem<<<1, 32>>>(da, db, np, dout); CK(cudaDeviceSynchronize());
  uint32_t ho[64]; CK(cudaMemcpy(ho, dout, np * 6 * 4, cudaMemcpyDeviceToHost));
  printf("semantics: a b -> max.NaN min.NaN max min max.f64(hi) min.f64(hi)\n");
  for (int i = 0; i < np; ++i) {
    uint32_t ab, bb; memcpy(&ab, &ha[i], 4); memcpy(&bb, &hb[i], 4);
    printf("SEM %08x %08x -> %08x %08x %08x %08x %08x %08x\n", ab, bb, ho[i*6], ho[i*6+1], ho[i*6+2], ho[i*6+3], ho[i*6+4], ho[i*6+5]);
  }
  float hv[32]; for (int i = 0; i < 32; ++i) hv[i] = (i & 1) ? 0.0f : -0.0f;
  CK(cudaMemcpy(da, hv, 128, cudaMemcpyHostToDevice));
  k_redux<<<1, 32>>>(da, dout); CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(ho, dout, 8, cudaMemcpyDeviceToHost));
  printf("REDUX mixed zeros: max %08x min %08x\n", ho[0], ho[1]);
  // ---- bandwidth
  size_t bytes = (size_t)1 << 30;
  float* buf; CK(cudaMalloc(&buf, bytes)); CK(cudaMemset(buf, 0, bytes));
  float* o; CK(cudaMalloc(&o, 64));
  int sms = p.multiProcessorCount;
  const int blocks[] = {256, 512, 1024};
  for (int bi = 0; bi < 3; ++bi) {
    int B = blocks[bi];
    for (int occ = 1; occ <= 2048 / B * 2; occ *= 2) {
      int G = sms * occ;
      if ((size_t)G * B > 2048 * sms) continue;
      float t;
      t = time_kernel(k_bw<32, 4>, G, B, buf, bytes / 32, o, 20);
      printf("BW v8 U4 B=%4d G=%5d : %8.1f GB/s\n", B, G, bytes / t / 1e6);
      t = time_kernel(k_bw<32, 2>, G, B, buf, bytes / 32, o, 20);
      printf("BW v8 U2 B=%4d G=%5d : %8.1f GB/s\n", B, G, bytes / t / 1e6);
      t = time_kernel(k_bw<32, 8>, G, B, buf, bytes / 32, o, 20);
      printf("BW v8 U8 B=%4d G=%5d : %8.1f GB/s\n", B, G, bytes / t / 1e6);
      t = time_kernel(k_bw<16, 4>, G, B, buf, bytes / 16, o, 20);
      printf("BW v4 U4 B=%4d G=%5d : %8.1f GB/s\n", B, G, bytes / t / 1e6);
      t = time_kernel(k_bw<16, 8>, G, B, buf, bytes / 16, o, 20);
      printf("BW v4 U8 B=%4d G=%5d : %8.1f GB/s\n", B, G, bytes / t / 1e6);
      t = time_kernel(k_bw_tile<4>, G, B, buf, bytes / 32, o, 20);
      printf("BW tile v8 U4 B=%4d G=%5d : %8.1f GB/s\n", B, G, bytes / t / 1e6);
    }
  }
  // many-wave grids
  for (int G : {sms * 16, sms * 64, (int)(bytes / 32 / 256 / 4)}) {
    float t = time_kernel(k_bw<32, 4>, G, 256, buf, bytes / 32, o, 20);
    printf("BW v8 U4 B=256 G=%7d : %8.1f GB/s\n", G, bytes / t / 1e6);
  }
  // copy reference
  float* buf2; CK(cudaMalloc(&buf2, bytes));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaMemcpy(buf2, buf, bytes, cudaMemcpyDeviceToDevice);
  cudaEventRecord(e0);
  for (int r = 0; r < 10; ++r) cudaMemcpy(buf2, buf, bytes, cudaMemcpyDeviceToDevice);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  printf("memcpy D2D: %8.1f GB/s (read+write)\n", 2.0 * bytes * 10 / ms / 1e6);
  return 0;
}
