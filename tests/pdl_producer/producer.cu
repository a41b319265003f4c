// producer.cu -- TEST ONLY: a "foreign" kernel that writes a reduction's input
// after triggering its dependents early (griddepcontrol.launch_dependents at
// its very start, as cuBLAS / CUTLASS kernels do), then spins for `delay`
// cycles before storing.  Launched programmatically itself (pdl = 1) it first
// waits for its own primary (griddepcontrol.wait), as a well-formed
// programmatic secondary must before writing what the previous kernel reads.  A programmatically launched consumer may therefore
// start while these stores are still pending: it must execute
// griddepcontrol.wait before reading them (tests/test_early_loads_gpu.py).
#include <cuda_runtime.h>

__global__ void k_produce(int* x, long long n, int value, long long delay) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const long long t0 = clock64();
  while (clock64() - t0 < delay) {
  }
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) x[i] = value;
}

extern "C" int producer_launch(void* x, long long n, int value, long long delay, void* stream, int pdl) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148, 1, 1);  // one wave: every CTA is resident and triggers at once
  cfg.blockDim = dim3(256, 1, 1);
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return (int)cudaLaunchKernelEx(&cfg, k_produce, (int*)x, n, value, delay);
}
