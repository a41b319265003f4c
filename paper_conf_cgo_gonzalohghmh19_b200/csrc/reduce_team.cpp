// reduce_team.cpp -- sharded reduction with the cross-GPU combine fused into
// the reduction kernel: no NCCL launch on the data path.
//
// Each rank owns a small device buffer (kTeamBufBytes).  The buffers are
// mapped into every member's address space -- CUDA IPC handles across processes
// (P2P over NVLink / NVSwitch between GPUs, or the same GPU), or plain pointers
// within one process -- and the block that finishes a rank's local reduction
// writes its raw value, each 4-byte word paired with the call's epoch, into
// every member's buffer, polls its own buffer until all k values carry the
// epoch and combines them in rank order (kernel side: team_exchange in
// reduce_kernels.cuh).  One launch per call (two for TWO_PASS); the exchange is
// a few peer stores and one poll, no fences and no collective launch.
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "reduce_runtime.h"

namespace rb {
namespace {

struct Team {
  int k = 0, rank = 0, device = 0;
  char* own = nullptr;
  std::vector<char*> bufs;
  std::vector<bool> ipc_opened;
  char** d_bufs = nullptr;
  bool connected = false;
  bool shared_gpu = false;  // some peer buffer lives on this member's GPU
  std::mutex mu;
};

int team_upload(Team* t) {
  t->bufs[t->rank] = t->own;
  t->shared_gpu = false;
  for (int j = 0; j < t->k; ++j) {
    if (j == t->rank) continue;
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, t->bufs[j]);
    if (e != cudaSuccess) return cuda_fail(e, "cudaPointerGetAttributes (team peer buffer)");
    if (a.device == t->device) t->shared_gpu = true;
  }
  cudaError_t e = cudaMemcpy(t->d_bufs, t->bufs.data(), sizeof(char*) * t->k, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return cuda_fail(e, "team pointer upload");
  t->connected = true;
  return REDUCE_OK;
}

}  // namespace
}  // namespace rb

using namespace rb;

extern "C" {

int reduce_team_create(void** team_out, int nranks, int rank, void* ipc_handle_out) {
  if (!team_out) return fail(REDUCE_ERR_INVALID_ARG, "team_out is NULL");
  if (nranks < 1 || nranks > kTeamMaxRanks || rank < 0 || rank >= nranks)
    return fail(REDUCE_ERR_INVALID_ARG, "need 1 <= nranks <= 256 and 0 <= rank < nranks");
  Team* t = new Team();
  t->k = nranks;
  t->rank = rank;
  t->bufs.assign(nranks, nullptr);
  t->ipc_opened.assign(nranks, false);
  cudaError_t e = cudaGetDevice(&t->device);
  if (e == cudaSuccess) e = cudaMalloc(&t->own, kTeamBufBytes);
  if (e == cudaSuccess) e = cudaMemset(t->own, 0, kTeamBufBytes);  // flags and counter start at 0
  if (e == cudaSuccess) e = cudaMalloc(&t->d_bufs, sizeof(char*) * nranks);
  if (e == cudaSuccess && ipc_handle_out) {
    cudaIpcMemHandle_t h;
    e = cudaIpcGetMemHandle(&h, t->own);
    if (e == cudaSuccess) std::memcpy(ipc_handle_out, &h, sizeof(h));
  }
  if (e != cudaSuccess) {
    if (t->own) cudaFree(t->own);
    if (t->d_bufs) cudaFree(t->d_bufs);
    delete t;
    return cuda_fail(e, "reduce_team_create");
  }
  *team_out = t;
  return REDUCE_OK;
}

int reduce_team_ipc_handle_bytes(void) { return (int)sizeof(cudaIpcMemHandle_t); }

void* reduce_team_buffer(void* team) { return team ? ((Team*)team)->own : nullptr; }

int reduce_team_connect(void* team, const void* handles) {
  if (!team || !handles) return fail(REDUCE_ERR_INVALID_ARG, "team / handles is NULL");
  Team* t = (Team*)team;
  std::lock_guard<std::mutex> lk(t->mu);
  for (int j = 0; j < t->k; ++j) {
    if (j == t->rank) continue;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, (const char*)handles + (size_t)j * sizeof(h), sizeof(h));
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle (team peer buffer)");
    t->bufs[j] = (char*)p;
    t->ipc_opened[j] = true;
  }
  return team_upload(t);
}

int reduce_team_connect_local(void* team, void* const* bufs) {
  if (!team || !bufs) return fail(REDUCE_ERR_INVALID_ARG, "team / bufs is NULL");
  Team* t = (Team*)team;
  std::lock_guard<std::mutex> lk(t->mu);
  for (int j = 0; j < t->k; ++j) {
    if (!bufs[j]) return fail(REDUCE_ERR_INVALID_ARG, "a team buffer pointer is NULL");
    if (j != t->rank) t->bufs[j] = (char*)bufs[j];
  }
  return team_upload(t);
}

int reduce_team_destroy(void* team) {
  if (!team) return fail(REDUCE_ERR_INVALID_ARG, "team is NULL");
  Team* t = (Team*)team;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(t->device);
  for (int j = 0; j < t->k; ++j)
    if (t->ipc_opened[j]) cudaIpcCloseMemHandle(t->bufs[j]);
  cudaFree(t->own);
  cudaFree(t->d_bufs);
  cudaSetDevice(prev);
  delete t;
  return REDUCE_OK;
}

int reduce_multi_team(int dtype, int op, const void* in_local, size_t n_local, void* out, reduce_stream_t stream,
                      void* team, const reduce_opts_t* opts) {
  if (out == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "out is NULL");
  if (team == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "team is NULL");
  Team* t = (Team*)team;
  if (!t->connected) return fail(REDUCE_ERR_INVALID_ARG, "team is not connected");
  const int s = (dtype == REDUCE_FLOAT64) ? 8 : 4;
  if (((uintptr_t)out % (uintptr_t)s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "out is not aligned to the element size");
  Plan P;
  int st = make_plan(dtype, op, in_local, n_local, opts, 0, &P);
  if (st != REDUCE_OK) return st;
  Workspace* ws = nullptr;
  if ((st = get_workspace_for((cudaStream_t)stream, P, &ws)) != REDUCE_OK) return st;
  {
    std::lock_guard<std::mutex> lk(t->mu);
    P.d.team.bufs = t->d_bufs;
    P.d.team.k = t->k;
    P.d.team.rank = t->rank;  // the epoch is advanced on the device (graph-capturable)
    P.d.team.shared_gpu = t->shared_gpu ? 1 : 0;
  }
  return launch_plan(&P, ws, out, (cudaStream_t)stream);
}

}  // extern "C"
