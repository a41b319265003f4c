// probe_mc.cu -- which cuMulticastCreate properties does this box accept for a
// one-device multicast team?  Not product code.
#include <cstdio>
#include <cstring>
#include <cuda.h>
#include <cuda_runtime.h>
template <class F> F get(const char* n) {
  void* f = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint(n, &f, cudaEnableDefault, &q);
  return (F)f;
}
int main() {
  cudaSetDevice(0);
  cudaFree(0);
  auto attr = get<decltype(&cuDeviceGetAttribute)>("cuDeviceGetAttribute");
  auto create = get<decltype(&cuMulticastCreate)>("cuMulticastCreate");
  auto gran = get<decltype(&cuMulticastGetGranularity)>("cuMulticastGetGranularity");
  int v = -1;
  attr(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, 0);
  printf("MULTICAST_SUPPORTED=%d\n", v);
  int fab = -1;
  attr(&fab, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, 0);
  printf("HANDLE_TYPE_FABRIC_SUPPORTED=%d\n", fab);
  unsigned long long hts[] = {0, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_FABRIC,
                              CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR | CU_MEM_HANDLE_TYPE_FABRIC};
  for (int nd = 1; nd <= 2; ++nd)
    for (auto ht : hts) {
      CUmulticastObjectProp p;
      memset(&p, 0, sizeof(p));
      p.numDevices = nd;
      p.size = 2 << 20;
      p.handleTypes = ht;
      size_t g = 0;
      CUresult rg = gran(&g, &p, CU_MULTICAST_GRANULARITY_RECOMMENDED);
      if (g) p.size = (p.size + g - 1) / g * g;
      CUmemGenericAllocationHandle h = 0;
      CUresult r = create(&h, &p);
      printf("numDevices=%d handleTypes=%llu gran=%zu (r=%d) create -> %d\n", nd, ht, g, (int)rg, (int)r);
    }
  return 0;
}
