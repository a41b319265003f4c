// Throwaway probe (not product code): what does a system-scope fence cost on
// B200?  One-thread kernels, 200 launches per CUDA graph, device time per
// launch.  Motivation: the team exchange (reduce_multi_team) added ~5 us per
// call at k=1 with two fence.acq_rel.sys.
#include <cstdio>
#include <cuda_runtime.h>

template <int V>
__global__ void k(unsigned* buf, unsigned e) {
  if (threadIdx.x != 0) return;
  if (V == 1) asm volatile("fence.acq_rel.gpu;" ::: "memory");
  if (V == 2) asm volatile("fence.acq_rel.sys;" ::: "memory");
  if (V == 3) asm volatile("fence.sc.sys;" ::: "memory");
  if (V == 4) asm volatile("fence.sc.gpu;" ::: "memory");
  if (V == 5) {  // store value, then release flag at sys scope, poll it back
    buf[16] = e;
    asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(buf), "r"(e) : "memory");
    unsigned v;
    do asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(buf) : "memory"); while (v != e);
  }
  if (V == 6) {  // LL-style: {data, flag} in one 8-byte store, relaxed poll
    asm volatile("st.relaxed.sys.global.v2.u32 [%0], {%1, %2};" :: "l"(buf + 32), "r"(e * 3), "r"(e) : "memory");
    unsigned d, f;
    do asm volatile("ld.relaxed.sys.global.v2.u32 {%0, %1}, [%2];" : "=r"(d), "=r"(f) : "l"(buf + 32) : "memory"); while (f != e);
    buf[48] = d;
  }
  if (V == 7) {  // volatile store + poll
    ((volatile unsigned*)buf)[64] = e;
    while (((volatile unsigned*)buf)[64] != e) {}
  }
  if (V == 8) __threadfence_system();
  if (V == 9) __threadfence();
}

template <int V>
float timeit(unsigned* buf, cudaStream_t s) {
  cudaGraph_t g; cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < 200; ++i) k<V><<<1, 32, 0, s>>>(buf, i + 1);
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(a, s);
    cudaGraphLaunch(ge, s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (r) best = ms * 1e3f / 200 < best ? ms * 1e3f / 200 : best;
  }
  return best;
}

int main() {
  unsigned* buf; cudaMalloc(&buf, 4096); cudaMemset(buf, 0, 4096);
  cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  printf("empty            %6.3f us\n", timeit<0>(buf, s));
  printf("fence.acq_rel.gpu %6.3f us\n", timeit<1>(buf, s));
  printf("fence.acq_rel.sys %6.3f us\n", timeit<2>(buf, s));
  printf("fence.sc.sys     %6.3f us\n", timeit<3>(buf, s));
  printf("fence.sc.gpu     %6.3f us\n", timeit<4>(buf, s));
  printf("rel/acq sys flag %6.3f us\n", timeit<5>(buf, s));
  printf("LL v2 relaxed    %6.3f us\n", timeit<6>(buf, s));
  printf("volatile flag    %6.3f us\n", timeit<7>(buf, s));
  printf("threadfence_sys  %6.3f us\n", timeit<8>(buf, s));
  printf("threadfence      %6.3f us\n", timeit<9>(buf, s));
  return 0;
}
