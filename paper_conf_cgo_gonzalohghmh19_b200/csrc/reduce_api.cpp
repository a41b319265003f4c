// reduce_api.cpp -- the C ABI of include/reduce.h: argument validation, the
// dispatch step (S0), the per-(device, stream) workspace, and error reporting.
// Every step of the reduction itself runs in the CUDA kernels; there is no
// host or CPU fallback anywhere in this library.
#include <atomic>
#include <climits>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <utility>

#include "reduce_runtime.h"

namespace rb {

struct DispatchEntry {
  int dtype, op, mode, max_log2_bytes, block, unroll, gc, bc, grid_cap, stage;  // stage 0 = registers
};
#include "dispatch_table.inc"

static thread_local std::string g_err;
static std::atomic<int> g_mode{REDUCE_MODE_FAST};
static std::mutex g_ws_mu;
// Workspaces are keyed by (device, CUDA stream id): cudaStreamPerThread has the
// same handle value in every host thread but names a different stream in each,
// and a destroyed stream's handle value may be reused by a new stream -- the
// id (cudaStreamGetId) is unique for both.
static std::map<std::pair<int, unsigned long long>, Workspace*> g_ws;

// cudaStreamGetId is not usable while the stream is being captured (it fails
// and would invalidate the capture), so the id seen by the last non-capturing
// call on a handle is cached: per host thread for the special handles (legacy
// default, per-thread default), process-wide for created streams.
static std::mutex g_sid_mu;
static std::map<cudaStream_t, unsigned long long> g_sid;
static thread_local std::map<cudaStream_t, unsigned long long> t_sid;

static unsigned long long stream_id(cudaStream_t s) {
  const bool special = (uintptr_t)s <= 2u;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  const bool capturing = cudaStreamIsCapturing(s, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone;
  if (!capturing) {
    unsigned long long id = 0;
    if (cudaStreamGetId(s, &id) == cudaSuccess) {
      if (special) {
        t_sid[s] = id;
      } else {
        std::lock_guard<std::mutex> lk(g_sid_mu);
        g_sid[s] = id;
      }
      return id;
    }
    cudaGetLastError();
  }
  if (special) {
    auto it = t_sid.find(s);
    if (it != t_sid.end()) return it->second;
  } else {
    std::lock_guard<std::mutex> lk(g_sid_mu);
    auto it = g_sid.find(s);
    if (it != g_sid.end()) return it->second;
  }
  return (unsigned long long)(uintptr_t)s | (1ull << 63);  // never seen outside a capture: no workspace yet
}

void set_error(const std::string& msg) { g_err = msg; }
int fail(int status, const std::string& msg) {
  g_err = msg;
  return status;
}
int cuda_fail(cudaError_t e, const char* what) {
  g_err = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
  return REDUCE_ERR_CUDA;
}
int default_mode() { return g_mode.load(); }

int num_sms() {
  int dev = 0, sms = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 148;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) return 148;
  return sms;
}

static int elem_bytes(int dtype) { return dtype == REDUCE_FLOAT64 ? 8 : 4; }
static int ilog2_ceil(unsigned long long v) {
  int l = 0;
  while ((1ull << l) < v && l < 63) ++l;
  return l;
}

int make_plan(int dtype, int op, const void* in, size_t n, const reduce_opts_t* opts, int raw_out, Plan* P) {
  if (dtype < 0 || dtype > 2) return fail(REDUCE_ERR_INVALID_ARG, "dtype must be REDUCE_INT32/FLOAT32/FLOAT64");
  if (op < 0 || op > 3) return fail(REDUCE_ERR_INVALID_ARG, "op must be REDUCE_SUM/MIN/MAX/SUM_ACCURATE");
  if (op == REDUCE_SUM_ACCURATE && dtype == REDUCE_INT32)
    return fail(REDUCE_ERR_INVALID_ARG, "REDUCE_SUM_ACCURATE needs a floating-point dtype (int32 sums are exact mod 2^32)");
  const int s = elem_bytes(dtype);
  if (n > 0 && in == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "in is NULL with n > 0");
  if (n > 0 && ((uintptr_t)in % (uintptr_t)s) != 0)
    return fail(REDUCE_ERR_INVALID_ARG, "in is not aligned to the element size");
  if (n > (size_t)1 << 46) return fail(REDUCE_ERR_INVALID_ARG, "n too large");

  reduce_opts_t o;
  o.mode = -1; o.grid_combine = -1; o.block_combine = -1; o.block = 0; o.unroll = 0; o.grid = 0; o.seg_group = 0;
  o.stage = 0; o.flags = 0;
  if (opts) o = *opts;
  if (o.flags & ~REDUCE_FLAG_INPUT_READY) return fail(REDUCE_ERR_INVALID_ARG, "unknown bits in flags");
  int mode = o.mode < 0 ? g_mode.load() : o.mode;
  if (mode != REDUCE_MODE_FAST && mode != REDUCE_MODE_DETERMINISTIC)
    return fail(REDUCE_ERR_INVALID_ARG, "mode must be -1, REDUCE_MODE_FAST or REDUCE_MODE_DETERMINISTIC");
  if (o.grid_combine < -1 || o.grid_combine > 5) return fail(REDUCE_ERR_INVALID_ARG, "bad grid_combine");
  if (o.block_combine < -1 || o.block_combine > 3) return fail(REDUCE_ERR_INVALID_ARG, "bad block_combine");
  if (o.unroll != 0 && o.unroll != 1 && o.unroll != 2 && o.unroll != 4 && o.unroll != 8 && o.unroll != 16)
    return fail(REDUCE_ERR_INVALID_ARG, "unroll must be 0, 1, 2, 4, 8 or 16");
  if (o.stage < 0 || o.stage > 2) return fail(REDUCE_ERR_INVALID_ARG, "stage must be 0, 1 or 2");
  if (o.block != 0 && (o.block < 32 || o.block > 1024 || o.block % 32 != 0))
    return fail(REDUCE_ERR_INVALID_ARG, "block must be 0 or a multiple of 32 in [32, 1024]");
  if (o.grid < -1) return fail(REDUCE_ERR_INVALID_ARG, "grid must be >= -1");
  if (mode == REDUCE_MODE_DETERMINISTIC) {
    if (o.grid_combine == REDUCE_GC_ATOMIC)
      return fail(REDUCE_ERR_INVALID_ARG, "deterministic mode forbids the ATOMIC grid combine");
    if (o.block_combine == REDUCE_BC_SMEM_ATOMIC_WARP || o.block_combine == REDUCE_BC_SMEM_ATOMIC_ALL)
      return fail(REDUCE_ERR_INVALID_ARG, "deterministic mode forbids shared-atomic block combines");
  }

  const bool dd = op == REDUCE_SUM_ACCURATE && dtype == REDUCE_FLOAT64;  // double-double: no atomics on values
  if (dd && o.grid_combine == REDUCE_GC_ATOMIC)
    return fail(REDUCE_ERR_INVALID_ARG, "fp64 accurate sums have no ATOMIC grid combine (double-double values)");
  if (dd && (o.block_combine == REDUCE_BC_SMEM_ATOMIC_WARP || o.block_combine == REDUCE_BC_SMEM_ATOMIC_ALL))
    return fail(REDUCE_ERR_INVALID_ARG, "fp64 accurate sums have no shared-atomic block combine");

  // ---- S0: table lookup by ceil(log2(bytes)); an op without tuned rows (the
  // accurate sum, if the table predates it) falls back to the sum rows.  The
  // first-match scan runs once per (dtype, op, mode, log2 bytes); its result
  // is cached (a pointer store: benign if two threads fill the same entry).
  // Calls with REDUCE_FLAG_INPUT_READY use their own tuned table (early
  // register loads make other launch shapes win), when one was generated.
  const unsigned long long bytes = (unsigned long long)n * (unsigned long long)s;
  const int lb = ilog2_ceil(bytes ? bytes : 1);
  const int ready = (kHaveReadyTable && (o.flags & REDUCE_FLAG_INPUT_READY)) ? 1 : 0;
  static std::atomic<const DispatchEntry*> cache[2][3][4][2][64];
  std::atomic<const DispatchEntry*>& slot = cache[ready][dtype][op][mode][lb & 63];
  const DispatchEntry* e = slot.load(std::memory_order_relaxed);
  if (e == nullptr) {
    const DispatchEntry* tab = ready ? kDispatchReady : kDispatch;
    const size_t rows = ready ? sizeof(kDispatchReady) / sizeof(kDispatchReady[0]) : sizeof(kDispatch) / sizeof(kDispatch[0]);
    for (int pass = 0; pass < 2 && (e == nullptr || e->dtype < 0); ++pass) {
      const int op_row = pass == 0 ? op : REDUCE_SUM;
      if (pass == 1 && op != REDUCE_SUM_ACCURATE) break;
      for (size_t i = 0; i < rows; ++i) {
        const DispatchEntry& r = tab[i];
        if ((r.dtype < 0 || r.dtype == dtype) && (r.op < 0 || r.op == op_row) && (r.mode < 0 || r.mode == mode) &&
            lb <= r.max_log2_bytes) {
          if (e == nullptr || r.dtype >= 0) e = &r;
          break;
        }
      }
    }
    if (!e) e = &tab[rows - 1];
    slot.store(e, std::memory_order_relaxed);
  }

  int stage = o.stage ? o.stage : (e->stage == REDUCE_STAGE_SMEM ? REDUCE_STAGE_SMEM : REDUCE_STAGE_REG);
  int block = o.block ? o.block : e->block;
  int unroll = o.unroll ? o.unroll : e->unroll;
  if (stage == REDUCE_STAGE_SMEM && !o.unroll && unroll < 4) unroll = 4;
  if (stage == REDUCE_STAGE_REG && !o.unroll && unroll > 8) unroll = 8;
  if (stage == REDUCE_STAGE_SMEM) {
    if (unroll != 4 && unroll != 8 && unroll != 16)
      return fail(REDUCE_ERR_INVALID_ARG, "shared-memory staging supports unroll 4, 8 or 16");
    if ((long long)block * unroll * 32 > kMaxSmemTileBytes)
      return fail(REDUCE_ERR_INVALID_ARG, "shared-memory tile (block*unroll*32) exceeds 128 KiB");
  } else if (unroll > 8) {
    return fail(REDUCE_ERR_INVALID_ARG, "register staging supports unroll 1, 2, 4 or 8");
  }
  int bc = o.block_combine >= 0 ? o.block_combine : e->bc;
  int gc;
  if (o.grid_combine >= 0) gc = o.grid_combine;
  else if (e->gc >= 0) gc = e->gc;
  else gc = mode == REDUCE_MODE_DETERMINISTIC ? REDUCE_GC_TWO_PASS : REDUCE_GC_ATOMIC;
  if (o.grid_combine < 0 && mode == REDUCE_MODE_DETERMINISTIC && gc == REDUCE_GC_ATOMIC) gc = REDUCE_GC_TWO_PASS;
  if (o.grid_combine < 0 && dd && gc == REDUCE_GC_ATOMIC) gc = REDUCE_GC_LAST_BLOCK;
  if (o.block_combine < 0 && (mode == REDUCE_MODE_DETERMINISTIC || dd) &&
      (bc == REDUCE_BC_SMEM_ATOMIC_WARP || bc == REDUCE_BC_SMEM_ATOMIC_ALL))
    bc = REDUCE_BC_SHFL;
  // grid: > 0 forced cap, -1 forced "one block per tile"; 0 takes the table's
  // cap, but only when the launch shape is the table's own (a cap tuned for
  // another block / unroll / staging would mis-shape a forced launch)
  const bool shape_forced = o.block || o.unroll || o.stage || o.grid_combine >= 0;
  const int grid_cap = o.grid > 0 ? o.grid : ((o.grid < 0 || shape_forced) ? 0 : e->grid_cap);
  if (!o.block && block > max_block_threads(dtype, op, unroll, stage)) block = max_block_threads(dtype, op, unroll, stage);
  if (block > max_block_threads(dtype, op, unroll, stage))
    return fail(REDUCE_ERR_INVALID_ARG, "block too large for this (dtype, op, unroll): max " +
                                            std::to_string(max_block_threads(dtype, op, unroll, stage)));
  if (bc == REDUCE_BC_SMEM_TREE && (block & (block - 1)) != 0)
    return fail(REDUCE_ERR_INVALID_ARG, "SMEM_TREE needs a power-of-two block");

  // ---- partition: head | 32-byte-aligned body of vectors | tail
  const int ve = 32 / s;
  size_t head = 0;
  if (n > 0) {
    const uintptr_t mis = (uintptr_t)in % 32u;
    head = mis ? (32u - mis) / (uintptr_t)s : 0;
    if (head > n) head = n;
  }
  const size_t rest = n - head;
  const unsigned long long body_vecs = rest / ve;
  const int tail = (int)(rest % ve);
  const long long tile_vecs = (long long)block * unroll;
  const long long tiles = (long long)((body_vecs + tile_vecs - 1) / tile_vecs);

  long long grid;
  if (gc == REDUCE_GC_DIRECT) {
    grid = 1;
  } else if (gc == REDUCE_GC_CLUSTER) {
    grid = grid_cap > 0 ? grid_cap : 16;
    if (grid > 16) return fail(REDUCE_ERR_INVALID_ARG, "cluster size must be <= 16");
    if (tiles > 0 && grid > tiles) grid = tiles;
  } else {
    grid = tiles > 0 ? tiles : 1;
    if (grid_cap > 0 && grid_cap < grid) grid = grid_cap;
    if ((gc == REDUCE_GC_TWO_PASS || gc == REDUCE_GC_LAST_BLOCK) && grid > kMaxPartialBlocks) grid = kMaxPartialBlocks;
    if (gc == REDUCE_GC_FLAGS && grid > kMaxFlagBlocks) grid = kMaxFlagBlocks;
    if (grid > 0x7FFFFFFFll) grid = 0x7FFFFFFFll;
  }
  int nslots = 0;  // ATOMIC: a power of two <= min(grid, 32) (the kernel masks, no modulo)
  if (gc == REDUCE_GC_ATOMIC)
    for (nslots = 1; nslots * 2 <= 32 && nslots * 2 <= grid;) nslots *= 2;

  // ---- longest fp addition chain L of this variant (for the G2 gate)
  long long chain = 0;
  if ((op == REDUCE_SUM || op == REDUCE_SUM_ACCURATE) && dtype != REDUCE_INT32) {
    const long long tpb = (tiles + grid - 1) / grid;
    const int nw = block / 32;
    if (op == REDUCE_SUM) {
      // vector tree (depth log2 VE) into 2 accumulators, +1 head/tail, +1 merging the two
      chain = (long long)((unroll + 1) / 2) * tpb + ilog2_ceil(32 / s) + 2;
    } else {
      const int na = dtype == REDUCE_FLOAT64 ? 4 : 8;  // one accumulator per vector lane
      chain = (long long)unroll * tpb + 1 + ilog2_ceil(na);
    }
    switch (bc) {
      case REDUCE_BC_SHFL: chain += 5 + (nw > 1 ? 5 : 0); break;
      case REDUCE_BC_SMEM_ATOMIC_WARP: chain += 5 + nw; break;
      case REDUCE_BC_SMEM_ATOMIC_ALL: chain += block; break;
      case REDUCE_BC_SMEM_TREE: chain += ilog2_ceil(block); break;
    }
    if (op == REDUCE_SUM_ACCURATE) {
      // the whole chain runs in fp64 (fp32 input) or double-double (fp64
      // input): L counts additions of that wider format, plus the final rounding
      switch (gc) {
        case REDUCE_GC_ATOMIC: chain += (grid + nslots - 1) / nslots + 5; break;
        case REDUCE_GC_TWO_PASS: chain += (grid + 255) / 256 + 2 + 10; break;
        case REDUCE_GC_LAST_BLOCK: chain += (grid + block - 1) / block + 2 + 10; break;
        case REDUCE_GC_FLAGS: chain += (grid + block - 1) / block + 10; break;  // per-thread run, 2 warp trees
        case REDUCE_GC_CLUSTER: chain += 5; break;
        default: break;
      }
    } else if (dtype == REDUCE_FLOAT32) {
      // blocks combine in fp64: the cross-block error is < grid * 2^-53 relative,
      // far below one fp32 ulp; the single fp64 -> fp32 rounding adds 1.
      chain += gc == REDUCE_GC_DIRECT ? 0 : 1;
    } else {
      switch (gc) {
        case REDUCE_GC_ATOMIC: chain += (grid + nslots - 1) / nslots + 5; break;
        case REDUCE_GC_TWO_PASS: chain += (grid + 255) / 256 + 2 + 10; break;
        case REDUCE_GC_LAST_BLOCK: chain += (grid + block - 1) / block + 2 + 10; break;
        case REDUCE_GC_FLAGS: chain += (grid + block - 1) / block + 10; break;  // per-thread run, 2 warp trees
        case REDUCE_GC_CLUSTER: chain += 5; break;
        default: break;
      }
    }
  }

  P->dtype = dtype; P->op = op; P->mode = mode; P->n = n; P->elem = s;
  P->input_ready = (o.flags & REDUCE_FLAG_INPUT_READY) != 0;
  LaunchDesc& d = P->d;
  std::memset(&d, 0, sizeof(d));
  d.dtype = dtype; d.op = op; d.in = in;
  d.body = (const char*)in + head * s;
  d.body_vecs = body_vecs; d.tiles = tiles;
  d.head = (int)head; d.tail = tail;
  d.grid = (int)grid; d.block = block; d.unroll = unroll; d.bc = bc; d.gc = gc; d.stage = stage;
  d.raw_out = raw_out; d.nslots = nslots;

  reduce_plan_t& p = P->pub;
  p.grid_combine = gc; p.block_combine = bc;
  p.grid = (int)grid; p.block = block; p.unroll = unroll; p.stage = stage;
  p.launches = gc == REDUCE_GC_TWO_PASS ? 2 : 1;
  p.slots = nslots; p.head = (int)head; p.tail = tail;
  p.tiles = tiles; p.chain = chain;
  return REDUCE_OK;
}

static void free_workspace(Workspace* w) {
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(w->device);
  if (w->base) cudaFree(w->base);
  if (w->partials) cudaFree(w->partials);
  if (w->flagrec) cudaFree(w->flagrec);
  if (w->segq) cudaFree(w->segq);
  if (w->segbal) cudaFree(w->segbal);
  if (w->staging) cudaFree(w->staging);
  for (int i = 0; i < 2; ++i) {
    if (w->ev_copied[i]) cudaEventDestroy(w->ev_copied[i]);
    if (w->ev_done[i]) cudaEventDestroy(w->ev_done[i]);
  }
  if (w->copy_stream) cudaStreamDestroy(w->copy_stream);
  cudaSetDevice(prev);
  delete w;
}

// REDUCE_FLAGS_EPOCH0 (tests only): the epoch a new record area starts from,
// so a test can cross the 32-bit wrap in a few calls
static unsigned flags_epoch0() {
  static const unsigned v = [] {
    const char* e = std::getenv("REDUCE_FLAGS_EPOCH0");
    return e ? (unsigned)std::strtoul(e, nullptr, 0) : 0u;
  }();
  return v;
}

int get_workspace(cudaStream_t stream, size_t partials_bytes, Workspace** out, size_t records_bytes) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
  const auto key = std::make_pair(dev, stream_id(stream));
  std::lock_guard<std::mutex> lk(g_ws_mu);
  Workspace*& w = g_ws[key];
  const bool need_base = (w == nullptr);
  const bool need_partials = (w == nullptr || w->partials_bytes < partials_bytes);
  const bool need_records = records_bytes > 0 && (w == nullptr || w->flagrec_bytes < records_bytes);
  if (need_base || need_partials || need_records) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(stream, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone) {
      if (need_base) g_ws.erase(key);
      return fail(REDUCE_ERR_NOT_PREPARED, "workspace missing or too small during stream capture: call reduce_prepare first");
    }
  }
  if (need_base) {
    Workspace* nw = new Workspace();
    nw->device = dev;
    nw->stream = stream;
    const size_t base_bytes = kCombos * kSlotRegionBytes + kCombos * (size_t)kSlotBytes + kNumScalars * kScalarBytes;
    e = cudaMalloc(&nw->base, base_bytes);
    if (e != cudaSuccess) {
      delete nw;
      g_ws.erase(key);
      cudaGetLastError();
      return fail(REDUCE_ERR_NO_MEMORY, "cudaMalloc(workspace) failed");
    }
    nw->slots = nw->base;
    nw->tickets = nw->base + kCombos * kSlotRegionBytes;
    nw->scalars = nw->tickets + kCombos * (size_t)kSlotBytes;
    e = launch_init_workspace(nw->slots, nw->tickets, stream);
    if (e != cudaSuccess) {
      cudaFree(nw->base);
      delete nw;
      g_ws.erase(key);
      return cuda_fail(e, "workspace init kernel");
    }
    w = nw;
  }
  if (w->partials_bytes < partials_bytes) {
    size_t want = partials_bytes < (64u << 10) ? (64u << 10) : partials_bytes;
    char* p = nullptr;
    // stream-ordered: the old buffer may still be read by queued kernels
    e = cudaMallocAsync((void**)&p, want, stream);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(REDUCE_ERR_NO_MEMORY, "cudaMallocAsync(partials) failed");
    }
    if (w->partials) cudaFreeAsync(w->partials, stream);
    w->partials = p;
    w->partials_bytes = want;
  }
  if (need_records) {
    size_t want = records_bytes < (64u << 10) ? (64u << 10) : records_bytes;
    char* p = nullptr;
    e = cudaMallocAsync((void**)&p, kFlagHdrBytes + want, stream);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(REDUCE_ERR_NO_MEMORY, "cudaMallocAsync(flag records) failed");
    }
    // zero records never match an epoch (epochs are >= 1); the header holds
    // the epoch and the record-area size (for the wrap, see flags_combine)
    e = cudaMemsetAsync(p, 0, kFlagHdrBytes + want, stream);
    struct { unsigned epoch, pad; unsigned long long bytes; } hdr = {flags_epoch0(), 0u, (unsigned long long)want};
    if (e == cudaSuccess) e = cudaMemcpyAsync(p, &hdr, sizeof(hdr), cudaMemcpyHostToDevice, stream);
    if (e != cudaSuccess) {
      cudaFreeAsync(p, stream);
      return cuda_fail(e, "flag records init");
    }
    if (w->flagrec) cudaFreeAsync(w->flagrec, stream);
    w->flagrec = p;
    w->flagrec_bytes = want;
  }
  *out = w;
  return REDUCE_OK;
}

// The stream's long-segment queue (allocated and zeroed on first use, or by
// reduce_prepare before a graph capture).
int get_seg_queue(cudaStream_t stream, char** out) {
  Workspace* w = nullptr;
  int st = get_workspace(stream, 0, &w);
  if (st != REDUCE_OK) return st;
  std::lock_guard<std::mutex> lk(g_ws_mu);
  if (w->segq == nullptr) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(stream, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone)
      return fail(REDUCE_ERR_NOT_PREPARED, "segment queue missing during stream capture: call reduce_prepare first");
    char* q = nullptr;
    cudaError_t e = cudaMalloc((void**)&q, kSegQBytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(REDUCE_ERR_NO_MEMORY, "cudaMalloc(segment queue) failed");
    }
    e = cudaMemsetAsync(q, 0, kSegQHdrBytes, stream);
    if (e != cudaSuccess) {
      cudaFree(q);
      return cuda_fail(e, "segment queue init");
    }
    w->segq = q;
  }
  *out = w->segq;
  return REDUCE_OK;
}

// The stream's chunk arrays of the element-balanced segmented path (allocated
// and its header zeroed on first use, or by reduce_prepare before a capture).
int get_seg_bal(cudaStream_t stream, char** out) {
  Workspace* w = nullptr;
  int st = get_workspace(stream, 0, &w);
  if (st != REDUCE_OK) return st;
  std::lock_guard<std::mutex> lk(g_ws_mu);
  if (w->segbal == nullptr) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(stream, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone)
      return fail(REDUCE_ERR_NOT_PREPARED, "segment chunk arrays missing during stream capture: call reduce_prepare first");
    char* b = nullptr;
    cudaError_t e = cudaMalloc((void**)&b, kBalBytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(REDUCE_ERR_NO_MEMORY, "cudaMalloc(segment chunk arrays) failed");
    }
    e = cudaMemsetAsync(b, 0, kBalHdrBytes, stream);
    if (e != cudaSuccess) {
      cudaFree(b);
      return cuda_fail(e, "segment chunk arrays init");
    }
    w->segbal = b;
  }
  *out = w->segbal;
  return REDUCE_OK;
}

int launch_plan(Plan* P, Workspace* ws, void* out, cudaStream_t stream, bool allow_early) {
  LaunchDesc& d = P->d;
  const int combo = combo_index(d.dtype, d.op);
  d.out = out;
  d.slots = ws->slots + combo * kSlotRegionBytes;
  d.ticket = (unsigned*)(ws->tickets + combo * (size_t)kSlotBytes);
  d.partials = ws->partials;
  if (d.gc == REDUCE_GC_FLAGS) {  // the epoch word and the records
    d.ticket = (unsigned*)ws->flagrec;
    d.partials = ws->flagrec + kFlagHdrBytes;
  }
  d.early = 0;
  // Before the programmatic dependency resolves a kernel may touch its input:
  //  1 = register loads of the first tile, only on the caller's explicit
  //      guarantee (REDUCE_FLAG_INPUT_READY) and when the input is not the
  //      previous library output -- a producer the library cannot see (a
  //      foreign kernel that triggered its dependents early) could still be
  //      writing it otherwise;
  //  2 = a bulk L2 prefetch of the first tile (always correct: a hint)
  if (early_enabled() && pdl_enabled() && P->n > 0) {
    d.early = prefetch_enabled() ? 2 : 0;
    if (allow_early && P->input_ready) {
      const uintptr_t lo = (uintptr_t)d.in, hi = lo + (uintptr_t)P->n * (uintptr_t)P->elem;
      if (hi <= ws->last_out_lo.load(std::memory_order_relaxed) || lo >= ws->last_out_hi.load(std::memory_order_relaxed))
        d.early = 1;
    }
  }
  cudaError_t e = launch_reduce(d, stream);
  if (allow_early) {  // this call wrote `out` only (one value of at most 16 bytes)
    ws->last_out_lo.store((uintptr_t)out, std::memory_order_relaxed);
    ws->last_out_hi.store((uintptr_t)out + 16, std::memory_order_relaxed);
  } else {
    ws->last_out_lo.store(0, std::memory_order_relaxed);
    ws->last_out_hi.store(~(uintptr_t)0, std::memory_order_relaxed);
  }
  if (e != cudaSuccess) return cuda_fail(e, "reduction kernel launch");
  return REDUCE_OK;
}

void note_unknown_output(cudaStream_t stream) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return;
  const auto key = std::make_pair(dev, stream_id(stream));
  std::lock_guard<std::mutex> lk(g_ws_mu);
  auto it = g_ws.find(key);
  if (it == g_ws.end() || it->second == nullptr) return;
  it->second->last_out_lo.store(0, std::memory_order_relaxed);
  it->second->last_out_hi.store(~(uintptr_t)0, std::memory_order_relaxed);
}

static size_t partials_needed(const Plan& P) {
  if (P.d.gc == REDUCE_GC_TWO_PASS || P.d.gc == REDUCE_GC_LAST_BLOCK)
    return (size_t)P.d.grid * (size_t)grid_value_bytes(P.dtype, P.op);
  return 0;
}

// GC_FLAGS: one record of 16-byte {word, epoch, word, epoch} stores per two
// words of the Grid value, per block
static size_t record_bytes(int dtype, int op) { return (size_t)((grid_value_bytes(dtype, op) + 7) / 8) * 16; }
static size_t records_needed(const Plan& P) {
  return P.d.gc == REDUCE_GC_FLAGS ? (size_t)P.d.grid * record_bytes(P.dtype, P.op) : 0;
}

int get_workspace_for(cudaStream_t stream, const Plan& P, Workspace** ws) {
  return get_workspace(stream, partials_needed(P), ws, records_needed(P));
}

}  // namespace rb

using namespace rb;

extern "C" {

int reduce_ex(int dtype, int op, const void* in, size_t n, void* out, reduce_stream_t stream,
              const reduce_opts_t* opts) {
  if (out == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "out is NULL");
  const int s = (dtype == REDUCE_FLOAT64) ? 8 : 4;
  if (((uintptr_t)out % (uintptr_t)s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "out is not aligned to the element size");
  Plan P;
  int st = make_plan(dtype, op, in, n, opts, 0, &P);
  if (st != REDUCE_OK) return st;
  Workspace* ws = nullptr;
  st = get_workspace_for((cudaStream_t)stream, P, &ws);
  if (st != REDUCE_OK) return st;
  return launch_plan(&P, ws, out, (cudaStream_t)stream, /*allow_early=*/true);
}

#ifndef RB_TILED_AUTO_MIN_LV
#define RB_TILED_AUTO_MIN_LV (-5)
#endif
static constexpr int kTiledAutoMinLv = RB_TILED_AUTO_MIN_LV;

static int segmented_common(int dtype, int op, const void* in, const int64_t* offsets, size_t seg_len,
                            size_t nseg, void* out, reduce_stream_t stream, const reduce_opts_t* opts) {
  if (dtype < 0 || dtype > 2) return fail(REDUCE_ERR_INVALID_ARG, "dtype must be REDUCE_INT32/FLOAT32/FLOAT64");
  if (op < 0 || op > 3) return fail(REDUCE_ERR_INVALID_ARG, "op must be REDUCE_SUM/MIN/MAX/SUM_ACCURATE");
  if (op == REDUCE_SUM_ACCURATE && dtype == REDUCE_INT32)
    return fail(REDUCE_ERR_INVALID_ARG, "REDUCE_SUM_ACCURATE needs a floating-point dtype");
  const int s = dtype == REDUCE_FLOAT64 ? 8 : 4;
  if (nseg == 0) return REDUCE_OK;
  if (out == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "out is NULL");
  note_unknown_output((cudaStream_t)stream);  // its kernels write `out` and trigger dependents early
  if (((uintptr_t)out % (uintptr_t)s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "out is not aligned to the element size");
  const bool uniform = offsets == nullptr;
  if (in == nullptr && (!uniform || seg_len > 0)) return fail(REDUCE_ERR_INVALID_ARG, "in is NULL");
  if (in && ((uintptr_t)in % (uintptr_t)s) != 0) return fail(REDUCE_ERR_INVALID_ARG, "in is not aligned to the element size");
  int block = 256, group = 0;
  if (opts) {
    if (opts->block != 0 && (opts->block < 32 || opts->block > 512 || opts->block % 32 != 0))
      return fail(REDUCE_ERR_INVALID_ARG, "segmented block must be 0 or a multiple of 32 in [32, 512]");
    if (opts->seg_group < 0 || opts->seg_group > 6) return fail(REDUCE_ERR_INVALID_ARG, "seg_group must be 0..6");
    if (opts->seg_group == 5 && uniform) return fail(REDUCE_ERR_INVALID_ARG, "seg_group 5 (balanced) needs an offsets array");
    if (opts->seg_group == 6 && !uniform) return fail(REDUCE_ERR_INVALID_ARG, "seg_group 6 (tiled rows) is for reduce_batched");
    if (opts->block) block = opts->block;
    group = opts->seg_group;
  }
  // auto: by row bytes for uniform batches (B200 sweep, tools/seg_bench.py);
  // element-balanced chunks for offset arrays (reduce_segbal.cuh), else 8
  // lanes (long segments go to the queue either way)
  const bool want_bal = !uniform && (group == 0 || group == 5) && nseg < 0xFFFFFFFFull;
  if (want_bal) {
    char* b = nullptr;
    if (get_seg_bal((cudaStream_t)stream, &b) == REDUCE_OK) {  // else (capture without prepare): group kernels
      SegParams p{};
      p.in = (const char*)in;
      p.offsets = (const long long*)offsets;
      p.nseg = (long long)nseg;
      p.out = out;
      p.balanced = 1;
      p.b = seg_bal_at(b);
      cudaError_t e = launch_segmented(dtype, op, p, 0, 0, (cudaStream_t)stream);
      if (e != cudaSuccess) return cuda_fail(e, "segmented reduction launch");
      return REDUCE_OK;
    }
  }
  if (group == 5) group = 3;
  const unsigned long long row_bytes = (unsigned long long)seg_len * (unsigned long long)s;
  // uniform rows of 32 B x 2^k (up to 32 KB) on 32-byte boundaries: the flat
  // kernel's 32 KB tile walk (k_rows_tiled); seg_group 6 asks for it, auto takes
  // it unless REDUCE_NO_ROWS_TILED=1
  int tiled_lv = -6;  // log2(row vectors) - 5 of an eligible row, -6: none
  if (uniform && in != nullptr && ((uintptr_t)in % 32u) == 0)
    for (int lv = -5; lv <= 5; ++lv)
      if (row_bytes == (32ull << (lv + 5))) tiled_lv = lv;
  // longer rows of whole 32 KB tiles, when there are enough of them to fill the
  // GPU with one block per row (B200 A/B, profiles/r01_rows_big_ab.jsonl: 0-19 %
  // faster from 2048 rows, up to 7 % slower at 1024 rows of 256 KB, where the
  // group kernels and the chunk queue keep their place)
  long long tiled_big = 0;
  if (uniform && in != nullptr && ((uintptr_t)in % 32u) == 0 && row_bytes >= (64u << 10) &&
      row_bytes % (32u << 10) == 0 && nseg >= 2048)
    tiled_big = (long long)(row_bytes / 32u);
  if (group == 6 && tiled_lv < -5 && tiled_big == 0)
    return fail(REDUCE_ERR_INVALID_ARG, "seg_group 6 needs 32-byte-aligned rows of 32 B x 2^k up to 32 KB, "
                                        "or >= 2048 rows of a multiple of 32 KB");
  // auto: rows of >= 2^(kTiledAutoMinLv + 5) vectors (measured: profiles/r01_rows_tiled_ab.jsonl,
  // profiles/r01_rows_small_ab.jsonl)
  // (every row size wins 1.05-1.75x, except accurate fp32 sums of 128-512 B rows:
  // 0.94-0.96x, those keep the one-thread-per-row kernel)
  const bool acc_f32_mid = op == REDUCE_SUM_ACCURATE && dtype == REDUCE_FLOAT32 && tiled_lv >= -3 && tiled_lv <= -1;
  const bool auto_tiled = ((tiled_lv >= kTiledAutoMinLv && !acc_f32_mid) || tiled_big > 0) && rows_tiled_enabled();
  if ((tiled_lv >= -5 || tiled_big > 0) && (group == 6 || (group == 0 && auto_tiled))) {
    SegParams p{};
    p.in = (const char*)in;
    p.seg_len = (long long)seg_len;
    p.nseg = (long long)nseg;
    p.out = out;
    p.rows_tiled = tiled_lv >= -5 ? 6 + tiled_lv : 12;
    p.rows_tiled_vecs = tiled_lv >= -5 ? 0 : tiled_big;
    cudaError_t e = launch_segmented(dtype, op, p, 0, 0, (cudaStream_t)stream);
    if (e != cudaSuccess) return cuda_fail(e, "segmented reduction launch");
    return REDUCE_OK;
  }
  if (group == 0)
    group = !uniform ? 3 : (row_bytes <= 512 ? 4 : (row_bytes <= 4096 ? 3 : (row_bytes <= 16384 ? 1 : 2)));
  const int lanes = group == 1 ? 32 : (group == 3 ? 8 : (group == 4 ? 1 : 0));
  SegParams p{};
  p.in = (const char*)in;
  p.offsets = (const long long*)offsets;
  p.seg_len = (long long)seg_len;
  p.nseg = (long long)nseg;
  p.out = out;
  p.raw_out = 0;
  // long-segment queue.  Offset arrays: always (lengths unknown here; a few
  // long segments would otherwise keep a few groups busy after the rest of
  // the GPU is done: power-law lengths 0.3 -> 1.5 TB/s on B200).  The
  // thresholds stay high -- queueing segments of a few KB (tried: 2 KB for 8
  // lanes) costs more than it balances.  Uniform rows are balanced by
  // construction: only when there are too few rows to fill the GPU.
  const long long ve = 32 / s;
  const long long first_round = lanes > 0 ? lanes : block;
  const long long long_vecs = lanes == 1 ? 32 : lanes == 8 ? 512 : lanes == 32 ? 2048 : 8192;
  const bool may_long = !uniform || ((long long)(seg_len / ve) > first_round + long_vecs - 1 && nseg < 4096 &&
                                     row_bytes > (64u << 10));
  p.use_q = 0;
  p.q = SegQueue{nullptr, nullptr, nullptr, nullptr};
  // uniform rows of whole 32-byte vectors on 32-byte boundaries, up to 256
  // bytes, one thread per row: every load of a row in flight at once
  if (uniform && lanes == 1 && in != nullptr && ((uintptr_t)in % 32u) == 0 && row_bytes > 0 &&
      row_bytes % 32u == 0 && row_bytes <= 256 && !(op == REDUCE_SUM_ACCURATE && row_bytes == 32))
    p.rows_nv = (int)(row_bytes / 32u);
  if (may_long && p.rows_nv == 0) {
    char* q = nullptr;
    if (get_seg_queue((cudaStream_t)stream, &q) == REDUCE_OK) {  // else (capture without prepare): no queue
      p.use_q = 1;
      p.q = seg_queue_at(q);
    }
  }
  cudaError_t e = launch_segmented(dtype, op, p, lanes, block, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "segmented reduction launch");
  return REDUCE_OK;
}

int reduce_segmented(int dtype, int op, const void* in, const int64_t* offsets, size_t num_segments, void* out,
                     reduce_stream_t stream, const reduce_opts_t* opts) {
  if (offsets == nullptr && num_segments > 0) return fail(REDUCE_ERR_INVALID_ARG, "offsets is NULL");
  return segmented_common(dtype, op, in, offsets, 0, num_segments, out, stream, opts);
}

int reduce_batched(int dtype, int op, const void* in, size_t seg_len, size_t num_segments, void* out,
                   reduce_stream_t stream, const reduce_opts_t* opts) {
  return segmented_common(dtype, op, in, nullptr, seg_len, num_segments, out, stream, opts);
}

int reduce_histogram(int dtype, const void* in, size_t n, double lo, double hi, int nbins, uint32_t* counts,
                     reduce_stream_t stream) {
  if (dtype != REDUCE_INT32 && dtype != REDUCE_FLOAT32)
    return fail(REDUCE_ERR_INVALID_ARG, "histogram input must be REDUCE_INT32 or REDUCE_FLOAT32");
  if (nbins < 1 || nbins > (1 << 24)) return fail(REDUCE_ERR_INVALID_ARG, "nbins must be in [1, 2^24]");
  if (!(lo < hi) || !std::isfinite(lo) || !std::isfinite(hi)) return fail(REDUCE_ERR_INVALID_ARG, "need finite lo < hi");
  if (counts == nullptr || ((uintptr_t)counts % 4u) != 0) return fail(REDUCE_ERR_INVALID_ARG, "counts is NULL or misaligned");
  if (n > 0 && (in == nullptr || ((uintptr_t)in % 4u) != 0))
    return fail(REDUCE_ERR_INVALID_ARG, "in is NULL or not aligned to the element size");
  HistParams p = {};
  p.in = (const char*)in;
  size_t head = 0;
  if (n > 0) {
    const uintptr_t mis = (uintptr_t)in % 32u;
    head = mis ? (32u - mis) / 4u : 0;
    if (head > n) head = n;
  }
  p.body = (const char*)in + head * 4;
  p.body_vecs = (n - head) / 8;
  p.head = (int)head;
  p.tail = (int)((n - head) % 8);
  if (dtype == REDUCE_INT32) {
    if (lo != std::floor(lo) || hi != std::floor(hi) || lo < -4294967296.0 || hi > 4294967296.0)
      return fail(REDUCE_ERR_INVALID_ARG, "int32 histograms need integer lo, hi within +-2^32");
    p.lo_i = (long long)lo;
    p.hi_i = (long long)hi;
    p.range_i = (unsigned long long)(p.hi_i - p.lo_i);
    p.magic = ~0ull / p.range_i;
    const long long lo_c = p.lo_i > (long long)INT32_MIN ? p.lo_i : (long long)INT32_MIN;
    const long long hi_c = p.hi_i < (long long)INT32_MAX + 1 ? p.hi_i : (long long)INT32_MAX + 1;
    p.narrow = ((unsigned long long)p.range_i * (unsigned long long)nbins < (1ull << 32) && hi_c > lo_c) ? 1 : 0;
    // q = (t + ((n - t) >> 1)) >> shift32, t = umulhi(n, magic32): with
    // l = ceil(log2 d), magic32 = floor(2^32 (2^l - d) / d) + 1, shift32 = l - 1
    // (Granlund & Montgomery 1994, fig. 4.1).  d = 1: every counted element
    // has n = 0, which the zero multiplier maps to 0.
    p.magic32 = 0u;
    p.shift32 = 0;
    if (p.narrow && p.range_i > 1) {
      int l = 0;
      while ((1ull << l) < p.range_i) ++l;
      const unsigned __int128 num = ((unsigned __int128)1 << 32) * ((1ull << l) - p.range_i);
      p.magic32 = (unsigned)(num / p.range_i + 1);
      p.shift32 = l - 1;
    }
    p.lo_c32 = (unsigned)(long long)lo_c;
    p.lim32 = p.narrow ? (unsigned)(hi_c - 1 - lo_c) : 0u;
    p.lo32 = (unsigned)p.lo_i;
  } else {
    p.lo_f = (float)lo;
    p.hi_f = (float)hi;
    p.scale_f = (float)((double)nbins / (hi - lo));
  }
  p.nbins = nbins;
  p.counts = counts;
  p.merge64 = ((uintptr_t)counts % 8u) == 0 && (unsigned long long)n < (1ull << 32);
  note_unknown_output((cudaStream_t)stream);
  cudaError_t e = launch_histogram(dtype, p, 256, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "histogram launch");
  return REDUCE_OK;
}

int reduce(int dtype, int op, const void* in, size_t n, void* out, reduce_stream_t stream) {
  return reduce_ex(dtype, op, in, n, out, stream, nullptr);
}

int reduce_query_plan(int dtype, int op, const void* in, size_t n, const reduce_opts_t* opts, reduce_plan_t* plan) {
  if (plan == nullptr) return fail(REDUCE_ERR_INVALID_ARG, "plan is NULL");
  Plan P;
  // `in` is only used for alignment here; allow NULL by treating it as aligned
  const void* probe = in ? in : (const void*)(uintptr_t)256;
  int st = make_plan(dtype, op, probe, n, opts, 0, &P);
  if (st != REDUCE_OK) return st;
  *plan = P.pub;
  return REDUCE_OK;
}

int reduce_prepare(reduce_stream_t stream, size_t max_n) {
  // partials for the largest partials-based grid any call of up to max_n
  // elements can plan: the smallest tile is 32 threads x 1 vector = 128
  // elements (fp64; 256 for 4-byte types), the widest cross-block value is 16
  // bytes (fp64 accurate sums: double-double), the grid is capped at
  // kMaxPartialBlocks
  const unsigned long long tiles_min_tile = (max_n + 127) / 128;
  long long g = (long long)(tiles_min_tile < (unsigned long long)kMaxPartialBlocks ? tiles_min_tile : kMaxPartialBlocks);
  if (g < 1024) g = 1024;
  Workspace* ws = nullptr;
  const long long gf = g < kMaxFlagBlocks ? g : kMaxFlagBlocks;
  int st = get_workspace((cudaStream_t)stream, (size_t)g * 16, &ws, (size_t)gf * 32);
  if (st != REDUCE_OK) return st;
  char* q = nullptr;
  st = get_seg_queue((cudaStream_t)stream, &q);  // so segmented calls can be captured too
  if (st != REDUCE_OK) return st;
  char* b = nullptr;
  st = get_seg_bal((cudaStream_t)stream, &b);
  if (st != REDUCE_OK) return st;
  if (cudaMemsetAsync(b, 0, kBalHdrBytes, (cudaStream_t)stream) != cudaSuccess) return cuda_fail(cudaGetLastError(), "segment chunk arrays reset");
  // queue counters back to zero too (recovery after an aborted segmented call)
  cudaError_t e = cudaMemsetAsync(q, 0, kSegQHdrBytes, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "segment queue reset");
  e = launch_init_workspace(ws->slots, ws->tickets, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "workspace init kernel");
  return REDUCE_OK;
}

void reduce_set_mode(int mode) {
  if (mode == REDUCE_MODE_FAST || mode == REDUCE_MODE_DETERMINISTIC) g_mode.store(mode);
}
int reduce_get_mode(void) { return g_mode.load(); }

const char* reduce_status_string(int status) {
  switch (status) {
    case REDUCE_OK: return "REDUCE_OK";
    case REDUCE_ERR_INVALID_ARG: return "REDUCE_ERR_INVALID_ARG";
    case REDUCE_ERR_UNSUPPORTED: return "REDUCE_ERR_UNSUPPORTED";
    case REDUCE_ERR_CUDA: return "REDUCE_ERR_CUDA";
    case REDUCE_ERR_NCCL: return "REDUCE_ERR_NCCL";
    case REDUCE_ERR_NO_MEMORY: return "REDUCE_ERR_NO_MEMORY";
    case REDUCE_ERR_NOT_PREPARED: return "REDUCE_ERR_NOT_PREPARED";
  }
  return "REDUCE_ERR_UNKNOWN";
}

const char* reduce_last_error(void) { return g_err.c_str(); }

int reduce_version(void) { return 10000 * 0 + 100 * 1 + 0; }

void reduce_shutdown(void) {
  std::lock_guard<std::mutex> lk(g_ws_mu);
  // the stream a workspace was made for may be gone (or be another thread's
  // per-thread stream): wait for each device instead
  for (auto& kv : g_ws) {
    if (kv.second) {
      int prev = 0;
      cudaGetDevice(&prev);
      cudaSetDevice(kv.second->device);
      cudaDeviceSynchronize();
      cudaSetDevice(prev);
      free_workspace(kv.second);
    }
  }
  cudaGetLastError();
  g_ws.clear();
}

}  // extern "C"
