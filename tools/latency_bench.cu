// latency_bench.cu -- host-side cost of one reduce() call through the C ABI
// (no Python): for small n (BASELINE configs[3], 32-64K elements) it reports
//   launch_us : host time inside reduce() (validation, dispatch, launch),
//   wall_us   : reduce() + cudaStreamSynchronize (what a caller waits for),
//   graph_us  : device time per call inside a CUDA graph of 100 calls.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -I include \
//          tools/latency_bench.cu -o tools/latency_bench -L<pkg> -lreduce_b200 -Xlinker -rpath,<pkg>
#include <chrono>
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
#include "reduce.h"

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  const size_t max_n = 1 << 16;
  int* din;
  float* dfin;
  void* dout;
  cudaMalloc(&din, max_n * 4 * 128);
  cudaMalloc(&dfin, max_n * 4 * 128);
  cudaMalloc(&dout, 1 << 12);
  cudaMemset(din, 0, max_n * 4 * 128);
  cudaMemset(dfin, 0, max_n * 4 * 128);
  reduce_prepare((reduce_stream_t)s, max_n);
  printf("{\"latency\": [");
  bool first = true;
  for (int dt = 0; dt < 2; ++dt) {
    const void* base = dt == 0 ? (const void*)din : (const void*)dfin;
    for (size_t n : {32ul, 256ul, 1024ul, 4096ul, 16384ul, 65536ul}) {
      std::vector<double> launch, wall;
      for (int i = 0; i < 200; ++i) {
        const void* in = (const char*)base + (size_t)(i % 64) * n * 4;
        double t0 = now_us();
        int st = reduce(dt, REDUCE_SUM, in, n, dout, (reduce_stream_t)s);
        double t1 = now_us();
        cudaStreamSynchronize(s);
        double t2 = now_us();
        if (st) { printf("error %s\n", reduce_last_error()); return 1; }
        if (i >= 20) { launch.push_back(t1 - t0); wall.push_back(t2 - t0); }
      }
      std::sort(launch.begin(), launch.end());
      std::sort(wall.begin(), wall.end());
      cudaGraph_t g;
      cudaGraphExec_t ge;
      cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
      for (int i = 0; i < 100; ++i) reduce(dt, REDUCE_SUM, (const char*)base + (size_t)(i % 64) * n * 4, n, dout, (reduce_stream_t)s);
      cudaStreamEndCapture(s, &g);
      cudaGraphInstantiate(&ge, g, 0);
      cudaGraphLaunch(ge, s);
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a, s);
      cudaGraphLaunch(ge, s);
      cudaEventRecord(b, s);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      printf("%s{\"dtype\": \"%s\", \"n\": %zu, \"launch_us\": %.2f, \"wall_us\": %.2f, \"graph_us\": %.3f}",
             first ? "" : ", ", dt == 0 ? "int32" : "float32", n, launch[launch.size() / 2], wall[wall.size() / 2],
             ms * 1e3 / 100);
      first = false;
      cudaGraphExecDestroy(ge);
      cudaGraphDestroy(g);
    }
  }
  printf("]}\n");
  return 0;
}
