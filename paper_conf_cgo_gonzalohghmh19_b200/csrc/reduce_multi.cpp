// reduce_multi.cpp -- sharded mode (step S7 of DESIGN.md): every rank reduces
// its own shard with the single-GPU path, then the per-rank scalars are
// combined by ONE NCCL collective of one element over NVLink / NVSwitch.
//
// The paper is single-GPU (sec. IV); this is the north star's
// "8xB200 sharded mode ... combined with one NCCL allreduce".  The message is
// 4-8 bytes, so the collective is latency-bound (NCCL's LL protocol).
//
// NCCL is resolved at run time with dlopen("libnccl.so.2"): inside a process
// that imported torch this returns the very NCCL torch loaded, so the
// communicator and torch's process groups share one library.
#include <dlfcn.h>
#include <cstring>
#include <mutex>
#include <string>

#include <nccl.h>

#include "reduce_runtime.h"

namespace rb {
namespace {

struct NcclApi {
  bool tried = false, ok = false;
  decltype(&::ncclGetUniqueId) GetUniqueId = nullptr;
  decltype(&::ncclCommInitRank) CommInitRank = nullptr;
  decltype(&::ncclCommDestroy) CommDestroy = nullptr;
  decltype(&::ncclCommCount) CommCount = nullptr;
  decltype(&::ncclAllReduce) AllReduce = nullptr;
  decltype(&::ncclAllGather) AllGather = nullptr;
  decltype(&::ncclGetErrorString) GetErrorString = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

bool load_nccl() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.tried) return g_nccl.ok;
  g_nccl.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);  // torch's, if loaded
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    set_error(std::string("dlopen(libnccl.so.2) failed: ") + dlerror());
    return false;
  }
#define RB_SYM(field, name)                                                 \
  g_nccl.field = reinterpret_cast<decltype(g_nccl.field)>(dlsym(h, name)); \
  if (!g_nccl.field) {                                                      \
    set_error("libnccl.so.2 lacks " name);                                  \
    return false;                                                           \
  }
  RB_SYM(GetUniqueId, "ncclGetUniqueId");
  RB_SYM(CommInitRank, "ncclCommInitRank");
  RB_SYM(CommDestroy, "ncclCommDestroy");
  RB_SYM(CommCount, "ncclCommCount");
  RB_SYM(AllReduce, "ncclAllReduce");
  RB_SYM(AllGather, "ncclAllGather");
  RB_SYM(GetErrorString, "ncclGetErrorString");
#undef RB_SYM
  g_nccl.ok = true;
  return true;
}

int nccl_fail(ncclResult_t r, const char* what) {
  set_error(std::string(what) + ": " + (g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "?"));
  return REDUCE_ERR_NCCL;
}

// NCCL type of the raw (Grid) per-rank value, and the matching reduction.
// int32 sums travel as uint32 (wraparound is defined); fp32 sums as the fp64
// block-combine value; fp min/max as order-preserving unsigned keys.
ncclDataType_t raw_type(int dtype, int op) {
  if (dtype == REDUCE_INT32) return op == REDUCE_SUM ? ncclUint32 : ncclInt32;
  if (dtype == REDUCE_FLOAT32) return (op == REDUCE_SUM || op == REDUCE_SUM_ACCURATE) ? ncclFloat64 : ncclUint32;
  return (op == REDUCE_SUM || op == REDUCE_SUM_ACCURATE) ? ncclFloat64 : ncclUint64;
}
ncclRedOp_t raw_op(int op) {
  return (op == REDUCE_SUM || op == REDUCE_SUM_ACCURATE) ? ncclSum : (op == REDUCE_MIN ? ncclMin : ncclMax);
}

}  // namespace
}  // namespace rb

using namespace rb;

extern "C" {

int reduce_comm_unique_id_bytes(void) { return NCCL_UNIQUE_ID_BYTES; }

int reduce_comm_get_unique_id(void* id_out) {
  if (!id_out) return fail(REDUCE_ERR_INVALID_ARG, "id_out is NULL");
  if (!load_nccl()) return REDUCE_ERR_UNSUPPORTED;
  ncclUniqueId id;
  ncclResult_t r = g_nccl.GetUniqueId(&id);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  std::memcpy(id_out, &id, sizeof(id));
  return REDUCE_OK;
}

int reduce_comm_init(void** comm_out, const void* id, int nranks, int rank) {
  if (!comm_out || !id) return fail(REDUCE_ERR_INVALID_ARG, "comm_out / id is NULL");
  if (nranks < 1 || rank < 0 || rank >= nranks) return fail(REDUCE_ERR_INVALID_ARG, "bad nranks / rank");
  if (!load_nccl()) return REDUCE_ERR_UNSUPPORTED;
  ncclUniqueId uid;
  std::memcpy(&uid, id, sizeof(uid));
  ncclComm_t c = nullptr;
  ncclResult_t r = g_nccl.CommInitRank(&c, nranks, uid, rank);
  if (r != ncclSuccess) return nccl_fail(r, "ncclCommInitRank");
  *comm_out = (void*)c;
  return REDUCE_OK;
}

int reduce_comm_destroy(void* comm) {
  if (!comm) return fail(REDUCE_ERR_INVALID_ARG, "comm is NULL");
  if (!load_nccl()) return REDUCE_ERR_UNSUPPORTED;
  ncclResult_t r = g_nccl.CommDestroy((ncclComm_t)comm);
  if (r != ncclSuccess) return nccl_fail(r, "ncclCommDestroy");
  return REDUCE_OK;
}

int reduce_comm_count(void* comm, int* nranks) {
  if (!comm || !nranks) return fail(REDUCE_ERR_INVALID_ARG, "comm / nranks is NULL");
  if (!load_nccl()) return REDUCE_ERR_UNSUPPORTED;
  ncclResult_t r = g_nccl.CommCount((ncclComm_t)comm, nranks);
  if (r != ncclSuccess) return nccl_fail(r, "ncclCommCount");
  return REDUCE_OK;
}

int reduce_multi_ex(int dtype, int op, const void* in_local, size_t n_local, void* out, reduce_stream_t stream,
                    void* comm, const reduce_opts_t* opts) {
  if (out == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "out is NULL");
  if (comm == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "comm is NULL");
  const int s = (dtype == REDUCE_FLOAT64) ? 8 : 4;
  if (((uintptr_t)out % (uintptr_t)s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "out is not aligned to the element size");
  // raw == final bits for int32 (all ops) and fp64 sum: reduce straight into
  // `out` and all-reduce it in place (2 launches); otherwise reduce into a raw
  // workspace scalar, all-reduce it, and finalise with a one-warp kernel.
  const bool direct = dtype == REDUCE_INT32 || (dtype == REDUCE_FLOAT64 && op == REDUCE_SUM);
  Plan P;
  int st = make_plan(dtype, op, in_local, n_local, opts, direct ? 0 : 1, &P);
  if (st != REDUCE_OK) return st;
  if (!load_nccl()) return REDUCE_ERR_UNSUPPORTED;
  Workspace* ws = nullptr;
  st = get_workspace_for((cudaStream_t)stream, P, &ws);
  if (st != REDUCE_OK) return st;
  cudaStream_t cs = (cudaStream_t)stream;
  ncclComm_t c = (ncclComm_t)comm;
  const ncclDataType_t t = raw_type(dtype, op);
  void* raw = direct ? out : (void*)ws->scalars;

  // double-double raw values cannot be summed by NCCL: gather them instead
  const bool gather = P.mode == REDUCE_MODE_DETERMINISTIC || (dtype == REDUCE_FLOAT64 && op == REDUCE_SUM_ACCURATE);
  const size_t raw_count = (size_t)grid_value_bytes(dtype, op) / (t == ncclFloat64 || t == ncclUint64 ? 8 : 4);
  if (!gather) {
    if ((st = launch_plan(&P, ws, raw, cs)) != REDUCE_OK) return st;
    ncclResult_t r = g_nccl.AllReduce(raw, raw, 1, t, raw_op(op), c, cs);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllReduce");
    if (!direct) {
      cudaError_t e = launch_combine(dtype, op, raw, 1, out, 0, 32, cs);
      if (e != cudaSuccess) return cuda_fail(e, "finalise kernel");
    }
    return REDUCE_OK;
  }
  // deterministic: gather the raw per-rank values, combine them in rank order
  int nranks = 0;
  ncclResult_t r = g_nccl.CommCount(c, &nranks);
  if (r != ncclSuccess) return nccl_fail(r, "ncclCommCount");
  if ((size_t)nranks * 16 + kScalarBytes > (size_t)kNumScalars * kScalarBytes)
    return fail(REDUCE_ERR_UNSUPPORTED, "too many ranks for the deterministic gather buffer");
  P.d.raw_out = 1;
  raw = ws->scalars;
  void* gathered = ws->scalars + kScalarBytes;
  if ((st = launch_plan(&P, ws, raw, cs)) != REDUCE_OK) return st;
  r = g_nccl.AllGather(raw, gathered, raw_count, t, c, cs);
  if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather");
  cudaError_t e = launch_combine(dtype, op, gathered, nranks, out, 0, 32, cs);
  if (e != cudaSuccess) return cuda_fail(e, "rank-order combine kernel");
  return REDUCE_OK;
}

int reduce_multi(int dtype, int op, const void* in_local, size_t n_local, void* out, reduce_stream_t stream,
                 void* comm) {
  return reduce_multi_ex(dtype, op, in_local, n_local, out, stream, comm, nullptr);
}

}  // extern "C"
