// reduce_runtime.h -- host runtime internals shared by reduce_api.cpp,
// reduce_host.cpp and reduce_multi.cpp (not part of the ABI).
#pragma once
#include <atomic>
#include <cstdint>
#include <cstddef>
#include <cstdint>
#include <string>
#include <cuda_runtime.h>
#include "../../include/reduce.h"
#include "reduce_internal.h"

namespace rb {

// Per-(device, stream) workspace.  Everything is allocated once (or grown
// outside graph capture) and reused; the atomic slots reset themselves.
struct Workspace {
  int device = -1;
  cudaStream_t stream = nullptr;
  char* base = nullptr;        // slots | tickets | scalars
  char* slots = nullptr;       // kCombos regions of kSlotRegionBytes
  char* tickets = nullptr;     // kCombos words, kSlotBytes apart
  char* scalars = nullptr;     // 64 x 64-byte scratch scalars (raw results, gathers)
  char* partials = nullptr;    // per-block / per-chunk Grid values
  size_t partials_bytes = 0;
  // GC_FLAGS: [0, kFlagHdrBytes) header (u32 epoch at 0, u64 record-area bytes
  // at 8), then the flag-in-data records; never written by anything else, so a
  // stale record can only carry an older epoch
  char* flagrec = nullptr;
  size_t flagrec_bytes = 0;    // record area (excluding the header)
  char* segq = nullptr;        // long-segment queue of reduce_segmented / reduce_batched (kSegQBytes)
  char* segbal = nullptr;      // chunk arrays of the element-balanced reduce_segmented (kBalBytes)
  // device bytes the last library call on this stream wrote for the caller
  // ([0, max) = unknown): a reduce whose input does not overlap them may load
  // its first tile before its programmatic dependency resolves
  std::atomic<uintptr_t> last_out_lo{0}, last_out_hi{~(uintptr_t)0};
  // reduce_host staging (lazily created)
  char* staging = nullptr;     // 2 x staging_bytes
  size_t staging_bytes = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copied[2] = {nullptr, nullptr};
  cudaEvent_t ev_done[2] = {nullptr, nullptr};
};

constexpr size_t kScalarBytes = 64;
constexpr int kNumScalars = 64;
constexpr long long kMaxPartialBlocks = 1 << 16;  // grid cap for partials-based combines
constexpr long long kMaxFlagBlocks = 1 << 13;     // grid cap for GC_FLAGS (one block polls them all)
constexpr size_t kFlagHdrBytes = 256;

// Resolved plan of one reduction call (step S0).
struct Plan {
  int dtype, op, mode;
  size_t n;
  int elem;  // bytes per element
  bool input_ready;  // REDUCE_FLAG_INPUT_READY: early loads allowed (reduce / reduce_ex)
  LaunchDesc d;
  reduce_plan_t pub;
};

void set_error(const std::string& msg);
int fail(int status, const std::string& msg);
int cuda_fail(cudaError_t e, const char* what);

// Validate arguments (no CUDA calls) and resolve the launch.  `raw_out`
// selects the un-finalised Grid value as output.
int make_plan(int dtype, int op, const void* in, size_t n, const reduce_opts_t* opts, int raw_out,
              Plan* plan);

// Find or create the workspace for (current device, stream) with at least
// `partials_bytes` of partials and `records_bytes` of GC_FLAGS records.
// Returns REDUCE_ERR_NOT_PREPARED when an allocation would be needed during
// stream capture.
int get_workspace(cudaStream_t stream, size_t partials_bytes, Workspace** ws, size_t records_bytes = 0);
// The same, sized for one plan.
int get_workspace_for(cudaStream_t stream, const Plan& plan, Workspace** ws);

// Fill the workspace pointers of plan->d and launch it.  allow_early: a public
// single-array call (reduce / reduce_ex), whose written bytes are exactly
// `out`; other callers leave the stream's last output unknown.
int launch_plan(Plan* plan, Workspace* ws, void* out, cudaStream_t stream, bool allow_early = false);

// The stream's last output becomes unknown (entry points that launch other
// kernels: segmented, histogram).  No-op if the stream has no workspace yet.
void note_unknown_output(cudaStream_t stream);

int num_sms();
int default_mode();

}  // namespace rb
