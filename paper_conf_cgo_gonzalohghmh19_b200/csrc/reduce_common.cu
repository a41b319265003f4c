// reduce_common.cu -- dtype switch for the per-dtype kernel translation units.
#include <cstdlib>
#include "reduce_internal.h"

namespace rb {

cudaError_t launch_reduce_i32(const LaunchDesc&, cudaStream_t);
cudaError_t launch_reduce_f32(const LaunchDesc&, cudaStream_t);
cudaError_t launch_reduce_f64(const LaunchDesc&, cudaStream_t);
cudaError_t combine_i32(int, const void*, long long, void*, int, int, cudaStream_t, TeamArgs);
cudaError_t combine_f32(int, const void*, long long, void*, int, int, cudaStream_t, TeamArgs);
cudaError_t combine_f64(int, const void*, long long, void*, int, int, cudaStream_t, TeamArgs);
cudaError_t init_i32(char*, char*, cudaStream_t);
cudaError_t init_f32(char*, char*, cudaStream_t);
cudaError_t init_f64(char*, char*, cudaStream_t);
cudaError_t segmented_i32(int, const SegParams&, int, int, cudaStream_t);
cudaError_t segmented_f32(int, const SegParams&, int, int, cudaStream_t);
cudaError_t segmented_f64(int, const SegParams&, int, int, cudaStream_t);

cudaError_t histogram_i32(const HistParams&, int, cudaStream_t);
cudaError_t histogram_f32(const HistParams&, int, cudaStream_t);

cudaError_t launch_histogram(int dtype, const HistParams& p, int block, cudaStream_t s) {
  if (dtype == 0) return histogram_i32(p, block, s);
  if (dtype == 1) return histogram_f32(p, block, s);
  return cudaErrorInvalidValue;
}

cudaError_t launch_segmented(int dtype, int op, const SegParams& p, int group, int block, cudaStream_t s) {
  switch (dtype) {
    case 0: return segmented_i32(op, p, group, block, s);
    case 1: return segmented_f32(op, p, group, block, s);
    case 2: return segmented_f64(op, p, group, block, s);
  }
  return cudaErrorInvalidValue;
}

bool pdl_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("REDUCE_NO_PDL");
    return !(e && e[0] == '1');
  }();
  return on;
}

bool early_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("REDUCE_NO_EARLY");
    return !(e && e[0] == '1');
  }();
  return on;
}

bool prefetch_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("REDUCE_NO_PREFETCH");
    return !(e && e[0] == '1');
  }();
  return on;
}

long long prefetch_budget_bytes() {
  static const long long b = [] {
    const char* e = std::getenv("REDUCE_PREFETCH_MB");
    long long mb = e ? std::atoll(e) : 0;  // B200 A/B: deeper prefetch gains nothing (profiles/r02_prefetch_depth_ab.jsonl)
    return (mb < 0 ? 0 : mb) << 20;
  }();
  return b;
}

bool rows_tiled_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("REDUCE_NO_ROWS_TILED");
    return !(e && e[0] == '1');
  }();
  return on;
}

int grid_value_bytes(int dtype, int op) {
  if (dtype == 0) return 4;                                // int32: uint32 / int32
  if (dtype == 1) return (op == 0 || op == 3) ? 8 : 4;     // fp32: double sums / uint32 key
  return op == 3 ? 16 : 8;                                 // fp64: double-double / double / uint64 key
}

cudaError_t launch_reduce(const LaunchDesc& d, cudaStream_t s) {
  switch (d.dtype) {
    case 0: return launch_reduce_i32(d, s);
    case 1: return launch_reduce_f32(d, s);
    case 2: return launch_reduce_f64(d, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_combine(int dtype, int op, const void* vals, long long count, void* out, int raw_out,
                           int block, cudaStream_t s, TeamArgs team) {
  switch (dtype) {
    case 0: return combine_i32(op, vals, count, out, raw_out, block, s, team);
    case 1: return combine_f32(op, vals, count, out, raw_out, block, s, team);
    case 2: return combine_f64(op, vals, count, out, raw_out, block, s, team);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_init_workspace(void* slots_base, void* tickets_base, cudaStream_t s) {
  cudaError_t e;
  if ((e = init_i32((char*)slots_base, (char*)tickets_base, s)) != cudaSuccess) return e;
  if ((e = init_f32((char*)slots_base, (char*)tickets_base, s)) != cudaSuccess) return e;
  return init_f64((char*)slots_base, (char*)tickets_base, s);
}

}  // namespace rb
