// reduce_nvls.cu -- sharded reduction with the cross-GPU combine done by
// NVLink SHARP (NVLS) multicast, fused into the reduction kernel (SURVEY 8(f)
// N2: "NVLS / symmetric-memory one-shot cross-GPU combine ... multimem.ld_reduce
// ... ncclCommWindowRegister ... fused as the epilogue of the last block").
//
// Host side only (the kernel side is nvls_exchange in reduce_kernels.cuh).
// reduce_nvls_create, a collective over an NCCL communicator:
//   1. ncclMemAlloc a 2 MB buffer on every rank (multicast-capable physical
//      memory), zero it, and register it as a SYMMETRIC window
//      (ncclCommWindowRegister, NCCL_WIN_COLL_SYMMETRIC): every rank's copy is
//      mapped into every rank's address space (the "LSA" team: ranks that
//      reach each other's memory over NVLink / NVSwitch);
//   2. ncclDevCommCreate with lsaMultimem: NCCL binds the windows to an NVLS
//      multicast object; its multicast base address comes back in the device
//      communicator;
//   3. the unicast address of every rank's copy and the window's multicast
//      address are resolved here (the window descriptor is read from device
//      memory; the arithmetic is the one of ncclGetLsaPointer /
//      ncclGetLsaMultimemPointer in nccl_device/impl/core__funcs.h), so the
//      reduction kernel needs nothing from NCCL but two addresses.
// No multicast (one GPU, no NVSwitch, NCCL without NVLS, ranks spread over
// several NVLink domains): REDUCE_ERR_UNSUPPORTED, and everything allocated
// so far is released.  NCCL is dlopen'ed as in reduce_multi.cpp.
#include <dlfcn.h>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include <cuda.h>  // driver types for the single-GPU multicast team (entry points via cudaGetDriverEntryPoint)
#include <nccl.h>
#include <nccl_device.h>

#include "reduce_runtime.h"

namespace rb {
namespace {

struct NvlsApi {
  bool tried = false, ok = false;
  decltype(&::ncclMemAlloc) MemAlloc = nullptr;
  decltype(&::ncclMemFree) MemFree = nullptr;
  decltype(&::ncclCommWindowRegister) WindowRegister = nullptr;
  decltype(&::ncclCommWindowDeregister) WindowDeregister = nullptr;
  decltype(&::ncclDevCommCreate) DevCommCreate = nullptr;
  decltype(&::ncclDevCommDestroy) DevCommDestroy = nullptr;
  decltype(&::ncclCommCount) CommCount = nullptr;
  decltype(&::ncclCommUserRank) CommUserRank = nullptr;
  decltype(&::ncclGetErrorString) GetErrorString = nullptr;
};
NvlsApi g_api;
std::mutex g_api_mu;

bool load_api() {
  std::lock_guard<std::mutex> lk(g_api_mu);
  if (g_api.tried) return g_api.ok;
  g_api.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    set_error(std::string("dlopen(libnccl.so.2) failed: ") + dlerror());
    return false;
  }
#define RB_SYM(field, name)                                                   \
  g_api.field = reinterpret_cast<decltype(g_api.field)>(dlsym(h, name));      \
  if (!g_api.field) {                                                         \
    set_error("libnccl.so.2 lacks " name " (symmetric memory needs NCCL >= 2.28)"); \
    return false;                                                             \
  }
  RB_SYM(MemAlloc, "ncclMemAlloc");
  RB_SYM(MemFree, "ncclMemFree");
  RB_SYM(WindowRegister, "ncclCommWindowRegister");
  RB_SYM(WindowDeregister, "ncclCommWindowDeregister");
  RB_SYM(DevCommCreate, "ncclDevCommCreate");
  RB_SYM(DevCommDestroy, "ncclDevCommDestroy");
  RB_SYM(CommCount, "ncclCommCount");
  RB_SYM(CommUserRank, "ncclCommUserRank");
  RB_SYM(GetErrorString, "ncclGetErrorString");
#undef RB_SYM
  g_api.ok = true;
  return true;
}

int nccl_err(ncclResult_t r, const char* what, int status) {
  set_error(std::string(what) + ": " + (g_api.GetErrorString ? g_api.GetErrorString(r) : "?"));
  return status;
}

// The high 32 bits of a flat address advanced by delta (nccl::utility::add4G).
char* add4g(char* base, int delta4g) {
  const unsigned long long p = (unsigned long long)(uintptr_t)base;
  const unsigned hi = (unsigned)(p >> 32) + (unsigned)delta4g;
  return (char*)(uintptr_t)((p & 0xFFFFFFFFull) | ((unsigned long long)hi << 32));
}

struct Nvls {
  ncclComm_t comm = nullptr;
  int k = 0, rank = 0, device = 0, mode = 1;
  void* buf = nullptr;
  ncclWindow_t win = nullptr;
  ncclDevComm dc;
  bool have_dc = false;
  char* mc = nullptr;
  std::vector<char*> peers;
  char** d_peers = nullptr;  // [k] unicast copies, [k] multicast address, [k + 1] counters
  unsigned* d_ctr = nullptr;
  // single-GPU multicast team (reduce_nvls_create_local): driver-API objects
  bool local = false;
  CUmemGenericAllocationHandle mc_handle = 0, mem_handle = 0;
  bool bound = false;
  CUdeviceptr uc_va = 0, mc_va = 0;
  size_t bytes = 0;
};

// Driver entry points (the library links only the static CUDA runtime).
struct DrvApi {
  bool tried = false, ok = false;
  decltype(&::cuMulticastCreate) MulticastCreate = nullptr;
  decltype(&::cuMulticastGetGranularity) MulticastGetGranularity = nullptr;
  decltype(&::cuMulticastAddDevice) MulticastAddDevice = nullptr;
  decltype(&::cuMulticastBindMem) MulticastBindMem = nullptr;
  decltype(&::cuMulticastUnbind) MulticastUnbind = nullptr;
  decltype(&::cuMemCreate) MemCreate = nullptr;
  decltype(&::cuMemRelease) MemRelease = nullptr;
  decltype(&::cuMemAddressReserve) MemAddressReserve = nullptr;
  decltype(&::cuMemAddressFree) MemAddressFree = nullptr;
  decltype(&::cuMemMap) MemMap = nullptr;
  decltype(&::cuMemUnmap) MemUnmap = nullptr;
  decltype(&::cuMemSetAccess) MemSetAccess = nullptr;
  decltype(&::cuDeviceGetAttribute) DeviceGetAttribute = nullptr;
};
DrvApi g_drv;

bool load_drv() {
  std::lock_guard<std::mutex> lk(g_api_mu);
  if (g_drv.tried) return g_drv.ok;
  g_drv.tried = true;
#define RB_DRV(field, name)                                                                       \
  {                                                                                               \
    void* fn = nullptr;                                                                           \
    cudaDriverEntryPointQueryResult q;                                                            \
    if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) {        \
      cudaGetLastError();                                                                         \
      set_error("driver entry point " name " unavailable");                                       \
      return false;                                                                               \
    }                                                                                             \
    g_drv.field = reinterpret_cast<decltype(g_drv.field)>(fn);                                    \
  }
  RB_DRV(MulticastCreate, "cuMulticastCreate");
  RB_DRV(MulticastGetGranularity, "cuMulticastGetGranularity");
  RB_DRV(MulticastAddDevice, "cuMulticastAddDevice");
  RB_DRV(MulticastBindMem, "cuMulticastBindMem");
  RB_DRV(MulticastUnbind, "cuMulticastUnbind");
  RB_DRV(MemCreate, "cuMemCreate");
  RB_DRV(MemRelease, "cuMemRelease");
  RB_DRV(MemAddressReserve, "cuMemAddressReserve");
  RB_DRV(MemAddressFree, "cuMemAddressFree");
  RB_DRV(MemMap, "cuMemMap");
  RB_DRV(MemUnmap, "cuMemUnmap");
  RB_DRV(MemSetAccess, "cuMemSetAccess");
  RB_DRV(DeviceGetAttribute, "cuDeviceGetAttribute");
#undef RB_DRV
  g_drv.ok = true;
  return true;
}

void release(Nvls* v) {
  if (v->have_dc) g_api.DevCommDestroy(v->comm, &v->dc);
  if (v->win) g_api.WindowDeregister(v->comm, v->win);
  if (v->buf) g_api.MemFree(v->buf);
  if (v->local) {
    if (v->mc_va) {
      g_drv.MemUnmap(v->mc_va, v->bytes);
      g_drv.MemAddressFree(v->mc_va, v->bytes);
    }
    if (v->uc_va) {
      g_drv.MemUnmap(v->uc_va, v->bytes);
      g_drv.MemAddressFree(v->uc_va, v->bytes);
    }
    if (v->bound) g_drv.MulticastUnbind(v->mc_handle, (CUdevice)v->device, 0, v->bytes);
    if (v->mem_handle) g_drv.MemRelease(v->mem_handle);
    if (v->mc_handle) g_drv.MemRelease(v->mc_handle);
  }
  if (v->d_peers) cudaFree(v->d_peers);
  if (v->d_ctr) cudaFree(v->d_ctr);
  delete v;
}

}  // namespace
}  // namespace rb

using namespace rb;

// Counters and the kernel's pointer table (shared by both constructions).
static int finish_setup(Nvls* v) {
  cudaError_t e = cudaMalloc(&v->d_ctr, 16);
  if (e == cudaSuccess) e = cudaMemset(v->d_ctr, 0, 16);
  std::vector<char*> table(v->peers);
  table.push_back(v->mc);
  table.push_back((char*)v->d_ctr);
  if (e == cudaSuccess) e = cudaMalloc(&v->d_peers, sizeof(char*) * table.size());
  if (e == cudaSuccess) e = cudaMemcpy(v->d_peers, table.data(), sizeof(char*) * table.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  return e == cudaSuccess ? REDUCE_OK : cuda_fail(e, "nvls setup");
}

extern "C" {

int reduce_nvls_supported(void* comm) {
  if (!comm) return fail(REDUCE_ERR_INVALID_ARG, "comm is NULL");
  if (!load_api()) return REDUCE_ERR_UNSUPPORTED;
  int k = 0;
  ncclResult_t r = g_api.CommCount((ncclComm_t)comm, &k);
  if (r != ncclSuccess) return nccl_err(r, "ncclCommCount", REDUCE_ERR_NCCL);
  if (k < 2) return fail(REDUCE_ERR_UNSUPPORTED, "NVLS needs at least two ranks");
  if (k > kTeamMaxRanks) return fail(REDUCE_ERR_UNSUPPORTED, "more ranks than the exchange slots hold (256)");
  if (!load_drv()) return REDUCE_ERR_UNSUPPORTED;
  int dev = 0, mc = 0;
  cudaGetDevice(&dev);
  if (g_drv.DeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, (CUdevice)dev) != CUDA_SUCCESS || !mc)
    return fail(REDUCE_ERR_UNSUPPORTED, "this device has no multicast support");
  return REDUCE_OK;
}

int reduce_nvls_create(void** nvls_out, void* comm, int mode) {
  if (!nvls_out || !comm) return fail(REDUCE_ERR_INVALID_ARG, "nvls_out / comm is NULL");
  if (mode != 1 && mode != 2) return fail(REDUCE_ERR_INVALID_ARG, "mode must be 1 (multimem.ld_reduce) or 2 (multicast store)");
  *nvls_out = nullptr;
  {
    const int st = reduce_nvls_supported(comm);  // local checks: no collective is entered without them
    if (st != REDUCE_OK) return st;
  }
  Nvls* v = new Nvls();
  v->comm = (ncclComm_t)comm;
  v->mode = mode;
  cudaGetDevice(&v->device);
  ncclResult_t r = g_api.CommCount(v->comm, &v->k);
  if (r == ncclSuccess) r = g_api.CommUserRank(v->comm, &v->rank);
  if (r != ncclSuccess) {
    release(v);
    return nccl_err(r, "ncclCommCount / ncclCommUserRank", REDUCE_ERR_NCCL);
  }
  if (v->k > kTeamMaxRanks) {
    release(v);
    return fail(REDUCE_ERR_UNSUPPORTED, "more ranks than the exchange slots hold (256)");
  }
  // 1. symmetric window (collective)
  r = g_api.MemAlloc(&v->buf, kNvlsAllocBytes);
  if (r != ncclSuccess) {
    release(v);
    return nccl_err(r, "ncclMemAlloc", REDUCE_ERR_UNSUPPORTED);
  }
  cudaError_t e = cudaMemset(v->buf, 0, kNvlsAllocBytes);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    release(v);
    return cuda_fail(e, "nvls buffer init");
  }
  r = g_api.WindowRegister(v->comm, v->buf, kNvlsAllocBytes, &v->win, NCCL_WIN_COLL_SYMMETRIC);
  if (r != ncclSuccess) {
    v->win = nullptr;
    release(v);
    return nccl_err(r, "ncclCommWindowRegister (symmetric)", REDUCE_ERR_UNSUPPORTED);
  }
  // 2. device communicator with NVLS multicast on the LSA team (collective)
  ncclDevCommRequirements reqs;
  std::memset(&reqs, 0, sizeof(reqs));
  reqs.lsaMultimem = true;
  std::memset(&v->dc, 0, sizeof(v->dc));
  r = g_api.DevCommCreate(v->comm, &reqs, &v->dc);
  if (r != ncclSuccess) {
    release(v);
    return nccl_err(r, "ncclDevCommCreate (lsaMultimem)", REDUCE_ERR_UNSUPPORTED);
  }
  v->have_dc = true;
  if (v->dc.lsaSize != v->k || v->dc.lsaMultimem.mcBasePtr == nullptr) {
    const std::string why = "no NVLS multicast across all " + std::to_string(v->k) + " ranks (lsaSize " +
                            std::to_string(v->dc.lsaSize) + ", multicast base " +
                            (v->dc.lsaMultimem.mcBasePtr ? "set" : "null") + ")";
    release(v);
    return fail(REDUCE_ERR_UNSUPPORTED, why);
  }
  // 3. addresses: every rank's copy (unicast) and the multicast address
  ncclWindow_vidmem wv;
  e = cudaMemcpy(&wv, v->win, sizeof(wv), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) {
    release(v);
    return cuda_fail(e, "reading the window descriptor");
  }
  v->peers.resize(v->k);
  for (int j = 0; j < v->k; ++j) v->peers[j] = add4g(wv.lsaFlatBase, j * (int)wv.stride4G);
  v->mc = (char*)v->dc.lsaMultimem.mcBasePtr + (size_t)wv.mcOffset4K * 4096;
  const int st = finish_setup(v);
  if (st != REDUCE_OK) {
    release(v);
    return st;
  }
  *nvls_out = v;
  return REDUCE_OK;
}

int reduce_nvls_create_local(void** nvls_out, int mode) {
  if (!nvls_out) return fail(REDUCE_ERR_INVALID_ARG, "nvls_out is NULL");
  if (mode != 1 && mode != 2) return fail(REDUCE_ERR_INVALID_ARG, "mode must be 1 (multimem.ld_reduce) or 2 (multicast store)");
  *nvls_out = nullptr;
  if (!load_drv()) return REDUCE_ERR_UNSUPPORTED;
  Nvls* v = new Nvls();
  v->local = true;
  v->k = 1;
  v->rank = 0;
  v->mode = mode;
  cudaGetDevice(&v->device);
  int mc_ok = 0;
  if (g_drv.DeviceGetAttribute(&mc_ok, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, (CUdevice)v->device) != CUDA_SUCCESS ||
      !mc_ok) {
    release(v);
    return fail(REDUCE_ERR_UNSUPPORTED, "this device has no multicast support");
  }
  CUmulticastObjectProp mp;
  std::memset(&mp, 0, sizeof(mp));
  mp.numDevices = 1;
  mp.size = kNvlsAllocBytes;
  size_t gran = 0;
  if (g_drv.MulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS || gran == 0) {
    release(v);
    return fail(REDUCE_ERR_UNSUPPORTED, "cuMulticastGetGranularity failed");
  }
  v->bytes = (kNvlsAllocBytes + gran - 1) / gran * gran;
  mp.size = v->bytes;
  CUmemAllocationProp ap;
  std::memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = v->device;
  CUmemAccessDesc acc;
  std::memset(&acc, 0, sizeof(acc));
  acc.location = ap.location;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  const char* step = "cuMulticastCreate";
  CUresult r = g_drv.MulticastCreate(&v->mc_handle, &mp);
  if (r == CUDA_SUCCESS) { step = "cuMulticastAddDevice"; r = g_drv.MulticastAddDevice(v->mc_handle, (CUdevice)v->device); }
  if (r == CUDA_SUCCESS) { step = "cuMemCreate"; r = g_drv.MemCreate(&v->mem_handle, v->bytes, &ap, 0); }
  if (r == CUDA_SUCCESS) { step = "cuMulticastBindMem"; r = g_drv.MulticastBindMem(v->mc_handle, 0, v->mem_handle, 0, v->bytes, 0); }
  if (r == CUDA_SUCCESS) v->bound = true;
  if (r == CUDA_SUCCESS) { step = "cuMemAddressReserve"; r = g_drv.MemAddressReserve(&v->uc_va, v->bytes, gran, 0, 0); }
  if (r == CUDA_SUCCESS) { step = "cuMemMap"; r = g_drv.MemMap(v->uc_va, v->bytes, 0, v->mem_handle, 0); }
  if (r == CUDA_SUCCESS) { step = "cuMemSetAccess"; r = g_drv.MemSetAccess(v->uc_va, v->bytes, &acc, 1); }
  if (r == CUDA_SUCCESS) { step = "cuMemAddressReserve (mc)"; r = g_drv.MemAddressReserve(&v->mc_va, v->bytes, gran, 0, 0); }
  if (r == CUDA_SUCCESS) { step = "cuMemMap (mc)"; r = g_drv.MemMap(v->mc_va, v->bytes, 0, v->mc_handle, 0); }
  if (r == CUDA_SUCCESS) { step = "cuMemSetAccess (mc)"; r = g_drv.MemSetAccess(v->mc_va, v->bytes, &acc, 1); }
  if (r != CUDA_SUCCESS) {
    const std::string why = std::string("single-GPU multicast setup failed at ") + step + " (CUresult " +
                            std::to_string((int)r) + ")";
    release(v);
    return fail(REDUCE_ERR_UNSUPPORTED, why);
  }
  cudaError_t e = cudaMemset((void*)v->uc_va, 0, v->bytes);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    release(v);
    return cuda_fail(e, "multicast buffer init");
  }
  v->peers.assign(1, (char*)v->uc_va);
  v->mc = (char*)v->mc_va;
  const int st = finish_setup(v);
  if (st != REDUCE_OK) {
    release(v);
    return st;
  }
  *nvls_out = v;
  return REDUCE_OK;
}

int reduce_nvls_destroy(void* nvls) {
  if (!nvls) return fail(REDUCE_ERR_INVALID_ARG, "nvls is NULL");
  Nvls* v = (Nvls*)nvls;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(v->device);
  cudaDeviceSynchronize();
  release(v);
  cudaSetDevice(prev);
  return REDUCE_OK;
}

int reduce_multi_nvls(int dtype, int op, const void* in_local, size_t n_local, void* out, reduce_stream_t stream,
                      void* nvls, const reduce_opts_t* opts) {
  if (out == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "out is NULL");
  if (nvls == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "nvls is NULL");
  Nvls* v = (Nvls*)nvls;
  const int s = (dtype == REDUCE_FLOAT64) ? 8 : 4;
  if (((uintptr_t)out % (uintptr_t)s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "out is not aligned to the element size");
  Plan P;
  int st = make_plan(dtype, op, in_local, n_local, opts, 0, &P);
  if (st != REDUCE_OK) return st;
  Workspace* ws = nullptr;
  if ((st = get_workspace_for((cudaStream_t)stream, P, &ws)) != REDUCE_OK) return st;
  P.d.team.bufs = v->d_peers;
  P.d.team.k = v->k;
  P.d.team.rank = v->rank;
  P.d.team.shared_gpu = 0;
  // deterministic mode: the multicast store + rank-order combine (mode 2); the
  // switch's reduction order for fp sums is not specified
  P.d.team.nvls = (short)(P.mode == REDUCE_MODE_DETERMINISTIC ? 2 : v->mode);
  return launch_plan(&P, ws, out, (cudaStream_t)stream);
}

}  // extern "C"
