// reduce_f64.cu -- instantiates the reduction kernels for one dtype (split per
// dtype so the 48 kernel instantiations per dtype compile in parallel).
#include "reduce_kernels.cuh"
#include "reduce_segbal.cuh"

namespace rb {
cudaError_t launch_reduce_f64(const LaunchDesc& d, cudaStream_t s) { return launch_dt<DT_F64>(d, s); }
cudaError_t combine_f64(int op, const void* v, long long c, void* out, int raw, int block, cudaStream_t s, TeamArgs t) {
  return combine_dt<DT_F64>(op, v, c, out, raw, block, s, t);
}
cudaError_t init_f64(char* slots, char* tickets, cudaStream_t s) { return init_dt<DT_F64>(slots, tickets, s); }
cudaError_t segmented_f64(int op, const SegParams& p, int group, int block, cudaStream_t s) {
  if (p.balanced) return launch_segbal_dt<DT_F64>(op, p, s);
  return launch_segmented_dt<DT_F64>(op, p, group, block, s);
}
}  // namespace rb
