// reduce_f32.cu -- instantiates the reduction kernels for one dtype (split per
// dtype so the 48 kernel instantiations per dtype compile in parallel).
#include "reduce_kernels.cuh"
#include "reduce_segbal.cuh"
#include "reduce_histogram.cuh"

namespace rb {
cudaError_t launch_reduce_f32(const LaunchDesc& d, cudaStream_t s) { return launch_dt<DT_F32>(d, s); }
cudaError_t combine_f32(int op, const void* v, long long c, void* out, int raw, int block, cudaStream_t s, TeamArgs t) {
  return combine_dt<DT_F32>(op, v, c, out, raw, block, s, t);
}
cudaError_t init_f32(char* slots, char* tickets, cudaStream_t s) { return init_dt<DT_F32>(slots, tickets, s); }
cudaError_t segmented_f32(int op, const SegParams& p, int group, int block, cudaStream_t s) {
  if (p.balanced) return launch_segbal_dt<DT_F32>(op, p, s);
  return launch_segmented_dt<DT_F32>(op, p, group, block, s);
}
cudaError_t histogram_f32(const HistParams& p, int block, cudaStream_t s) {
  return launch_histogram_dt<DT_F32>(p, block, s);
}
}  // namespace rb
