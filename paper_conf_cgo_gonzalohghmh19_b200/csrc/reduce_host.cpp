// reduce_host.cpp -- end-to-end entry point with HOST buffers (the `e2e` leg
// of bench.py).  The input streams host -> device in chunks on a library copy
// stream while the previous chunk is reduced on the caller's stream (double
// buffering with events); each chunk leaves its raw (un-finalised) value in a
// device array, which one fixed-order combine kernel finalises, and a single
// element is copied back.  The paper excludes transfers from its timings
// (P:L641); this path exists so a user holding host data gets the whole job.
#include <cstring>
#include <string>

#include "reduce_runtime.h"

namespace rb {
namespace {
constexpr size_t kChunkBytes = 32u << 20;  // 32 MiB per staged chunk
constexpr long long kMaxChunks = 8192;
}  // namespace
}  // namespace rb

using namespace rb;

extern "C" int reduce_host(int dtype, int op, const void* host_in, size_t n, void* host_out, reduce_stream_t stream,
                           const reduce_opts_t* opts) {
  if (dtype < 0 || dtype > 2) return fail(REDUCE_ERR_INVALID_ARG, "dtype must be REDUCE_INT32/FLOAT32/FLOAT64");
  if (op < 0 || op > 3) return fail(REDUCE_ERR_INVALID_ARG, "op must be REDUCE_SUM/MIN/MAX/SUM_ACCURATE");
  if (host_out == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "host_out is NULL");
  if (n > 0 && host_in == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "host_in is NULL with n > 0");
  const size_t s = dtype == REDUCE_FLOAT64 ? 8 : 4;
  if (n > 0 && ((uintptr_t)host_in % s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "host_in is not aligned to the element size");
  cudaStream_t cs = (cudaStream_t)stream;

  size_t chunk_elems = kChunkBytes / s;
  long long nchunks = (long long)((n + chunk_elems - 1) / chunk_elems);
  if (nchunks > kMaxChunks) {
    chunk_elems = (n + kMaxChunks - 1) / kMaxChunks;
    chunk_elems = (chunk_elems + 7) / 8 * 8;  // keep chunks 32-byte aligned
    nchunks = (long long)((n + chunk_elems - 1) / chunk_elems);
  }
  const size_t chunk_bytes = chunk_elems * s;
  const int gbytes = grid_value_bytes(dtype, op);

  // plan of a full chunk (partials size for TWO_PASS / LAST_BLOCK)
  Plan P;
  int st = make_plan(dtype, op, (const void*)(uintptr_t)256, n < chunk_elems ? n : chunk_elems, opts, 1, &P);
  if (st != REDUCE_OK) return st;
  Workspace* ws = nullptr;
  if ((st = get_workspace_for(cs, P, &ws)) != REDUCE_OK) return st;

  // staging: 2 x chunk_bytes, then the per-chunk raw values
  const size_t vals_bytes = (size_t)kMaxChunks * 16;  // up to 16-byte raw values (double-double)
  if (ws->staging_bytes < chunk_bytes) {
    if (ws->staging) {
      cudaStreamSynchronize(cs);
      cudaFree(ws->staging);
      ws->staging = nullptr;
      ws->staging_bytes = 0;
    }
    cudaError_t e = cudaMalloc(&ws->staging, 2 * chunk_bytes + vals_bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(REDUCE_ERR_NO_MEMORY, "cudaMalloc(staging) failed");
    }
    ws->staging_bytes = chunk_bytes;
  }
  if (!ws->copy_stream) {
    cudaError_t e = cudaStreamCreateWithFlags(&ws->copy_stream, cudaStreamNonBlocking);
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
      e = cudaEventCreateWithFlags(&ws->ev_copied[i], cudaEventDisableTiming);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ws->ev_done[i], cudaEventDisableTiming);
    }
    if (e != cudaSuccess) return cuda_fail(e, "copy stream / events");
  }
  char* vals = ws->staging + 2 * ws->staging_bytes;
  cudaError_t e;
  for (long long c = 0; c < nchunks; ++c) {
    const int b = (int)(c & 1);
    const size_t off = (size_t)c * chunk_elems;
    const size_t cnt = (n - off) < chunk_elems ? (n - off) : chunk_elems;
    char* buf = ws->staging + (size_t)b * ws->staging_bytes;
    // the buffer is free once the kernel that read it (chunk c-2) is done
    if ((e = cudaStreamWaitEvent(ws->copy_stream, ws->ev_done[b], 0)) != cudaSuccess) return cuda_fail(e, "wait");
    if ((e = cudaMemcpyAsync(buf, (const char*)host_in + off * s, cnt * s, cudaMemcpyHostToDevice, ws->copy_stream)) !=
        cudaSuccess)
      return cuda_fail(e, "H2D chunk copy");
    if ((e = cudaEventRecord(ws->ev_copied[b], ws->copy_stream)) != cudaSuccess) return cuda_fail(e, "record");
    if ((e = cudaStreamWaitEvent(cs, ws->ev_copied[b], 0)) != cudaSuccess) return cuda_fail(e, "wait");
    Plan C;
    if ((st = make_plan(dtype, op, buf, cnt, opts, 1, &C)) != REDUCE_OK) return st;
    // the ragged last chunk may plan another grid combine than a full one
    if ((st = get_workspace_for(cs, C, &ws)) != REDUCE_OK) return st;
    if ((st = launch_plan(&C, ws, vals + (size_t)c * gbytes, cs)) != REDUCE_OK) return st;
    if ((e = cudaEventRecord(ws->ev_done[b], cs)) != cudaSuccess) return cuda_fail(e, "record");
  }
  if ((e = launch_combine(dtype, op, vals, nchunks, ws->scalars, 0, 256, cs)) != cudaSuccess)
    return cuda_fail(e, "chunk combine kernel");
  if ((e = cudaMemcpyAsync(host_out, ws->scalars, s, cudaMemcpyDeviceToHost, cs)) != cudaSuccess)
    return cuda_fail(e, "D2H result copy");
  if ((e = cudaStreamSynchronize(cs)) != cudaSuccess) return cuda_fail(e, "cudaStreamSynchronize");
  return REDUCE_OK;
}
