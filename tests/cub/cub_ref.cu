// cub_ref.cu -- TEST / BENCH CONTEXT ONLY (SURVEY 8(c) pin P10 and the paper's
// comparison baseline): cub::DeviceReduce from the CUDA 12.9 toolkit on
// the same device buffer.  Never linked into libreduce_b200.so.
//   cubref_reduce(dtype, op, in, n, out, stream) -> cudaError_t
//   dtype 0 int32, 1 fp32, 2 fp64; op 0 sum, 1 min, 2 max.
// Temporary storage is cached per process (grown on demand).
#include <cub/device/device_reduce.cuh>
#include <cuda_runtime.h>
#include <cstdint>

static void* g_tmp = nullptr;
static size_t g_tmp_bytes = 0;

template <class T>
static cudaError_t run(int op, const void* in, size_t n, void* out, cudaStream_t s) {
  const T* x = (const T*)in;
  T* o = (T*)out;
  size_t need = 0;
  cudaError_t e;
  auto call = [&](void* tmp, size_t& bytes) -> cudaError_t {
    if (op == 0) return cub::DeviceReduce::Sum(tmp, bytes, x, o, (int64_t)n, s);
    if (op == 1) return cub::DeviceReduce::Min(tmp, bytes, x, o, (int64_t)n, s);
    return cub::DeviceReduce::Max(tmp, bytes, x, o, (int64_t)n, s);
  };
  if ((e = call(nullptr, need)) != cudaSuccess) return e;
  if (need > g_tmp_bytes) {
    if (g_tmp) cudaFree(g_tmp);
    if ((e = cudaMalloc(&g_tmp, need)) != cudaSuccess) return e;
    g_tmp_bytes = need;
  }
  size_t bytes = g_tmp_bytes;
  return call(g_tmp, bytes);
}

extern "C" int cubref_reduce(int dtype, int op, const void* in, size_t n, void* out, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (dtype == 0) return (int)run<int32_t>(op, in, n, out, s);
  if (dtype == 1) return (int)run<float>(op, in, n, out, s);
  return (int)run<double>(op, in, n, out, s);
}
