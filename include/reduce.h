/*
 * reduce.h -- C ABI of libreduce_b200.so, a B200-native (sm_100a) device-wide
 * parallel reduction: one contiguous int32 / fp32 / fp64 array -> one scalar,
 * with op = sum, min or max.
 *
 * What the operation is (PAPER.md = the CGO'19 paper "Automatic Generation of
 * Warp-Level Primitives and Atomic Instructions for Fast and Portable Parallel
 * Reduction on GPUs"; citations P:Lnnn are its line numbers):
 *   - the spectrum `int sum(const Array<1,int> in)` returns one scalar, computed
 *     by the sequential codelet `accum += in[i]` (Fig. 1(a), sec. II.B.1);
 *   - the op set is the atomic Map API add / max / min (sec. III.A);
 *     `atomicSub` is not a reduction (not associative) and is not offered;
 *   - the host entry point takes the device input and leaves the result in
 *     device memory (Listing 1/2 `Reduce_Grid`).
 * How it is computed (steps S0-S7 of DESIGN.md): per-thread register
 * accumulation over 32-byte vector loads of a block-tiled / thread-strided
 * partition (Fig. 1(b)), a warp combine (shuffle / redux.sync,
 * Listing 4), a block combine (shared `partial[32]` "Vs", shared
 * atomics "VA1"/"VA2+S" Fig. 3, or a barrier'd shared tree "V"
 * Fig. 1(c)), and a grid combine (global atomics "DT,A" Listing 2, a
 * second kernel Listing 1, or a last-block pass).
 *
 * Conventions common to every entry point
 *   - Pointers: `in`/`out` are DEVICE pointers on the current CUDA device and
 *     are owned by the caller.  `out` receives exactly one element of the
 *     input's dtype and must not overlap `in`.  `in` must be aligned to the
 *     element size; any coarser misalignment is handled internally.
 *   - Asynchrony: every call is stream-ordered on `stream` and returns without
 *     host synchronisation (except reduce_host, see there).  The library owns
 *     only a small per-(device, stream) workspace, allocated on first use or by
 *     reduce_prepare(); calls are CUDA-graph capturable once prepared.
 *   - Errors: functions return a reduce_status_t.  Invalid arguments are
 *     rejected before any CUDA call is made.  Launch failures are reported as
 *     REDUCE_ERR_CUDA; asynchronous faults surface at the caller's next
 *     synchronisation, as in CUDA.  Nothing aborts, exits or throws across the
 *     ABI.  reduce_last_error() gives a thread-local detail message.
 *   - Semantics: int32 sum wraps modulo 2^32; fp sums
 *     accumulate in the element type within a block (fp32 block partials are
 *     combined across blocks in fp64); min/max are exact, NaN anywhere gives a
 *     canonical quiet NaN and -0.0 < +0.0; n == 0 writes the identity
 *     (0, INT32_MAX/+inf for min, INT32_MIN/-inf for max).
 *   - Determinism: REDUCE_MODE_DETERMINISTIC uses no atomic instruction at all
 *     (partials + a second kernel); its result bits depend only on
 *     (dtype, op, n, in % 32, SM count).  REDUCE_MODE_FAST combines blocks with
 *     global atomics: int32 and min/max results are still exact; fp sums may
 *     differ run to run in the last bits.
 */
#ifndef REDUCE_B200_H
#define REDUCE_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Same type as cudaStream_t (no CUDA header needed to use this ABI). NULL is
 * the legacy default stream. */
typedef struct CUstream_st* reduce_stream_t;

typedef enum { REDUCE_INT32 = 0, REDUCE_FLOAT32 = 1, REDUCE_FLOAT64 = 2 } reduce_dtype_t;
/* REDUCE_SUM_ACCURATE (fp dtypes only): the same sum at the
 * same bandwidth with a wider accumulator -- fp32 input accumulated in fp64 from
 * the first addition (error <= u_f|S| + (L+1)*2^-53*sum|x|), fp64 input in
 * double-double (Neumaier fold + TwoSum merges; error ~ u_d|S|).  The output
 * keeps the input dtype.  Beyond the paper, which reduces in the element type. */
typedef enum { REDUCE_SUM = 0, REDUCE_MIN = 1, REDUCE_MAX = 2, REDUCE_SUM_ACCURATE = 3 } reduce_op_t;
typedef enum { REDUCE_MODE_FAST = 0, REDUCE_MODE_DETERMINISTIC = 1 } reduce_mode_t;

typedef enum {
  REDUCE_OK = 0,
  REDUCE_ERR_INVALID_ARG = 1,  /* bad dtype/op/option, NULL or misaligned pointer */
  REDUCE_ERR_UNSUPPORTED = 2,  /* e.g. no sm_100 device, NCCL not loadable */
  REDUCE_ERR_CUDA = 3,         /* a CUDA runtime call or launch failed */
  REDUCE_ERR_NCCL = 4,         /* an NCCL call failed */
  REDUCE_ERR_NO_MEMORY = 5,    /* workspace allocation failed */
  REDUCE_ERR_NOT_PREPARED = 6  /* workspace missing/too small during graph capture */
} reduce_status_t;

/* Block combine (step S4), the paper's cooperative codelets:
 *   SHFL        "Vs"   : warp shuffle/redux -> shared partial[32] -> warp 0
 *                        (Fig. 1(c) after the shuffle pass, Listing 4)
 *   SMEM_ATOMIC_WARP "VA2+S": warp shuffle, lane 0 atomically combines into one
 *                        shared accumulator (Fig. 3(b), Listing 3)
 *   SMEM_ATOMIC_ALL  "VA1"  : every thread atomically combines into one shared
 *                        accumulator (Fig. 3(a))
 *   SMEM_TREE   "V"    : shared-memory tree with a barrier per step
 *                        (Fig. 1(c) lines 9-13) */
typedef enum {
  REDUCE_BC_SHFL = 0,
  REDUCE_BC_SMEM_ATOMIC_WARP = 1,
  REDUCE_BC_SMEM_ATOMIC_ALL = 2,
  REDUCE_BC_SMEM_TREE = 3
} reduce_block_combine_t;

/* Grid combine (step S5):
 *   DIRECT     : a single block writes the result (warp-only / single-block paths)
 *   ATOMIC     : "DT,A" -- one global atomic per block into a self-resetting
 *                accumulator, the last block (ticket) publishes it (Listing 2)
 *   TWO_PASS   : per-block partials + a second single-block kernel, no atomics
 *                (Listing 1 + second spectrum call)
 *   LAST_BLOCK : per-block partials; the last block (integer ticket) reduces
 *                them in a fixed order -- deterministic, one launch
 *   CLUSTER    : one thread-block cluster of `grid` CTAs (<= 16, on 16 SMs of
 *                one GPC) loops over all tiles; CTA partials meet in CTA 0's
 *                shared memory through distributed shared memory (DSMEM) and a
 *                cluster barrier -- no atomics, deterministic, one launch; the
 *                sm_90+/sm_100 form of the paper's two-stage per-SM partition
 *                 for medium arrays
 *   FLAGS      : every block but the last stores its partial with the call's
 *                epoch beside each 4-byte word (flag-in-data records); the
 *                last block polls them, reduces them in a fixed order and
 *                publishes -- no atomics, no fences, deterministic, one launch
 *                (a B200 design beside the paper's: one L2 round trip after the
 *                loads instead of ATOMIC's three; grid <= 8192 blocks) */
typedef enum {
  REDUCE_GC_DIRECT = 0,
  REDUCE_GC_ATOMIC = 1,
  REDUCE_GC_TWO_PASS = 2,
  REDUCE_GC_LAST_BLOCK = 3,
  REDUCE_GC_CLUSTER = 4,
  REDUCE_GC_FLAGS = 5
} reduce_grid_combine_t;

/* Options for reduce_ex & co.  Zero-initialise, then set fields; every field
 * has an "auto" value (-1 or 0) that takes the dispatch table's choice. */
typedef struct {
  int mode;           /* -1 = process default (reduce_set_mode), else reduce_mode_t */
  int grid_combine;   /* -1 = auto, else reduce_grid_combine_t */
  int block_combine;  /* -1 = auto, else reduce_block_combine_t */
  int block;          /* threads per block: 0 = auto, else 32..1024, multiple of 32
                         (power of two for SMEM_TREE) */
  int unroll;         /* 32-byte vectors per thread per tile: 0 = auto, else 1,2,4,8
                         (register staging) or 4,8,16 (shared-memory staging) */
  int grid;           /* 0 = auto (the dispatch table's grid cap when the launch shape
                         is also the table's, else one block per tile), -1 = one
                         block per tile, > 0 = at most this many blocks (persistent);
                         for REDUCE_GC_CLUSTER: the cluster size, 1..16 (0 = 16) */
  int seg_group;      /* reduce_segmented / reduce_batched only: 0 = auto (uniform
                         rows: one thread per row up to 512 bytes, 8 lanes up to 4 KB,
                         one warp up to 16 KB, else one block; offset arrays: the
                         element-balanced chunks of 5), 1 = one warp per segment,
                         2 = one block per segment, 3 = 8 lanes, 4 = one thread,
                         5 = element-balanced (offset arrays only): the elements are
                         cut into 4 KB chunks, each warp of a one-wave grid reduces a
                         contiguous range of chunks whatever the segment lengths, and
                         the segments crossing ranges are joined by a fix-up kernel
                         (3 launches; non-monotone offsets fall back to one warp per
                         segment inside the same launches).  For groups 1-4, segments
                         much longer than their group's first round (offset arrays; or
                         fewer than 4096 uniform rows of > 64 KB) are cut into chunks
                         of >= 16 KB that warps reduce (two more launches);
                         6 = tiled rows (reduce_batched only; 32-byte-aligned input,
                         rows of 32 B times a power of two up to 32 KB, or >= 2048 rows of
                         a multiple of 32 KB, else REDUCE_ERR_INVALID_ARG): each block
                         reads one contiguous 32 KB tile of whole rows, warp-loads are
                         reduced per row and combined in a fixed tree (longer rows: one
                         block per row walking its tiles) -- auto picks it for such
                         rows (except accurate fp32 sums of 128-512 B rows) unless
                         REDUCE_NO_ROWS_TILED=1 */
  int stage;          /* 0 = auto; REDUCE_STAGE_REG: 256-bit loads straight into
                         registers; REDUCE_STAGE_SMEM: cp.async 16-byte copies into a
                         shared-memory tile (block*unroll*32 <= 128 KiB), then shared
                         loads -- more bytes in flight per SM.  Same numerics. */
  int flags;          /* REDUCE_FLAG_* bits, 0 = none (reduce / reduce_ex only) */
} reduce_opts_t;

typedef enum { REDUCE_STAGE_AUTO = 0, REDUCE_STAGE_REG = 1, REDUCE_STAGE_SMEM = 2 } reduce_stage_t;

/* reduce_opts_t.flags:
 *   REDUCE_FLAG_INPUT_READY : the caller guarantees that no kernel that may
 *     still be running when this call is launched on `stream` writes `in`
 *     (e.g. the input was written before the previous kernel on the stream
 *     was launched, or was produced by another stream synchronised earlier).
 *     The reduction may then load its first tile before its programmatic
 *     dependency resolves ("early loads", see Stream ordering below). */
typedef enum { REDUCE_FLAG_INPUT_READY = 1 } reduce_flag_t;

/* What a call will launch (filled by reduce_query_plan). */
typedef struct {
  int grid_combine, block_combine;
  int grid, block, unroll, stage;
  int launches;        /* kernel launches per call: 1, or 2 for TWO_PASS */
  int slots;           /* global accumulator slots used by ATOMIC */
  int head, tail;      /* scalar elements before / after the 32-byte-aligned body */
  long long tiles;     /* B*unroll-vector tiles in the body */
  long long chain;     /* longest fp addition chain L (error bound (L+1)u*sum|x|) */
} reduce_plan_t;

/* Stream ordering.  Kernels are launched with programmatic dependent launch:
 * a reduction's first blocks may start while the previous kernel on the stream
 * drains, but by default they execute griddepcontrol.wait before touching any
 * memory, so the previous kernel's writes -- whoever launched it, and even if
 * it triggered its dependents early (griddepcontrol.launch_dependents, as
 * cuBLAS / CUTLASS kernels do) -- are complete and visible first.
 * Early loads are opt-in: with REDUCE_FLAG_INPUT_READY in reduce_opts_t.flags
 * (and an input that does not overlap the previous library call's output on
 * the stream) each block that is resident before the dependency resolves
 * loads its first tile of `in` before waiting.  That is only correct when the
 * caller's guarantee above holds; a producer kernel still writing `in` would
 * be read stale.  REDUCE_NO_EARLY=1 ignores the flag; REDUCE_NO_PDL=1 disables
 * programmatic launch altogether. */

/* Reduce in[0..n) with `op` into *out (device).  Uses the process-default mode. */
int reduce(int dtype, int op, const void* in, size_t n, void* out, reduce_stream_t stream);

/* As reduce(), with explicit mode / variant / launch overrides (opts may be NULL). */
int reduce_ex(int dtype, int op, const void* in, size_t n, void* out, reduce_stream_t stream,
              const reduce_opts_t* opts);

/* Describe what reduce_ex(dtype, op, in, n, ..., opts) would launch on the
 * current device.  `in` is only used for its address modulo 32 (may be any
 * value when n == 0).  No CUDA work is issued. */
int reduce_query_plan(int dtype, int op, const void* in, size_t n, const reduce_opts_t* opts,
                      reduce_plan_t* plan);

/* Allocate (or grow) the workspace of (current device, stream) so that calls
 * with up to `max_n` elements need no allocation -- call before graph capture.
 * Also allocates the stream's segment queue (reduce_segmented / reduce_batched;
 * a capture without it runs those calls without load balancing).
 * Also re-initialises the atomic accumulators and tickets (recovery after an
 * aborted kernel). */
int reduce_prepare(reduce_stream_t stream, size_t max_n);

void reduce_set_mode(int mode);  /* process-wide default for reduce(); invalid values ignored */
int reduce_get_mode(void);

/* End-to-end entry with HOST buffers: copies host_in (n elements; pinned memory
 * gives copy/compute overlap, pageable memory works but serialises) to the
 * device in chunks on `stream`, reduces each chunk while the next is in flight,
 * combines the chunk results on the device and copies the single result to
 * host_out.  Synchronises `stream` before returning, so *host_out is valid on
 * return.  Uses a library-owned device staging buffer (2 x chunk bytes). */
int reduce_host(int dtype, int op, const void* host_in, size_t n, void* host_out,
                reduce_stream_t stream, const reduce_opts_t* opts);

/* ---- many arrays in one launch ---------------------------
 * reduce_segmented: out[i] = reduce(in[offsets[i] .. offsets[i+1])) for every
 * i < num_segments.  `offsets` is a DEVICE array of num_segments + 1 int64
 * element offsets (non-decreasing; a decreasing pair is treated as an empty
 * segment, which yields the identity); `out` is a DEVICE array of
 * num_segments elements of dtype.  Offset arrays are reduced element-balanced
 * by default (seg_group 5: fixed 4 KB chunks of the flat element range, the
 * tiled partition of Fig. 1(b), with the segment boundaries carried
 * through it -- the time no longer depends on the length distribution);
 * the other groups give one thread, 8 lanes, one warp or one block per
 * segment (the paper's small-array versions assign one warp / block per
 * partition with no global atomics), and there segments much
 * longer than their group's first round are cut into chunks of >= 16 KB that
 * warps reduce, then combined in chunk order (the stream's workspace holds the
 * queue; two more launches).  Values never touch atomics and every combine
 * has a fixed order: deterministic.  Up to 3 launches (1 for uniform rows too
 * short to be cut).  num_segments must be < 2^32 - 1 for the balanced path
 * (else 8 lanes).  A graph capture needs reduce_prepare on the stream first
 * (the chunk arrays; without it the capture runs the group kernels).  Segment starts may have
 * any element alignment.  Options used: block (32..512, default 256), seg_group.  reduce_batched is the uniform case: num_segments rows of seg_len
 * contiguous elements (row i at in + i*seg_len), no offsets array. */
int reduce_segmented(int dtype, int op, const void* in, const int64_t* offsets, size_t num_segments, void* out,
                     reduce_stream_t stream, const reduce_opts_t* opts);
int reduce_batched(int dtype, int op, const void* in, size_t seg_len, size_t num_segments, void* out,
                   reduce_stream_t stream, const reduce_opts_t* opts);

/* ---- histogram -------------------------------------------
 * The workload the paper motivates shared-memory atomics with (P:L59,
 * P:L253-L255): counts[b] = #{ i : lo <= in[i] < hi and
 * b = floor((in[i] - lo) * nbins / (hi - lo)) }.  int32 input: lo and hi must
 * be integers (|.| <= 2^32) and the bin is exact integer arithmetic.  fp32
 * input: with lo_f = (float)lo, hi_f = (float)hi, scale = (float)(nbins/(hi-lo)),
 * x is counted iff lo_f <= x < hi_f, in bin floor(fl32(fl32(x - lo_f) * scale))
 * when that is in [0, nbins).  NaN is never counted.  `counts` is a DEVICE array of nbins uint32, overwritten (a memset
 * node precedes the kernel).  Per-block shared-memory histograms with
 * shared atomics (the paper's "VA1" codelet per bin), merged with global
 * atomics: up to 16384 bins as replicated 32-bit counters; up to what one
 * block's shared memory holds at 16 bits per bin (~116 K bins) in one pass
 * with 16-bit counters whose every 0x8000 is carried to `counts`; beyond that
 * in 16384-bin passes (up to 8), else straight into global memory.  Counts
 * are exact (integer atomics commute). */
int reduce_histogram(int dtype, const void* in, size_t n, double lo, double hi, int nbins, uint32_t* counts,
                     reduce_stream_t stream);

/* ---- sharded mode over NCCL (one process per GPU) -------------------------
 * reduce_multi: every rank of `comm` calls it with its own local shard
 * (n_local may differ per rank, and may be 0); each rank's local result is
 * combined with one in-place ncclAllReduce of a single element on `stream`
 * (fp min/max are combined as order-preserving integer keys so NaN / signed
 * zero semantics match the single-GPU path).  Every rank's *out receives the
 * global result.  In REDUCE_MODE_DETERMINISTIC the per-rank results are
 * all-gathered and combined in rank order by one warp instead (bitwise
 * reproducible for a fixed rank count).  `comm` is an ncclComm_t created by
 * reduce_comm_init (or borrowed from elsewhere; never destroyed here).
 * NCCL is loaded at run time (dlopen "libnccl.so.2"); without it these calls
 * return REDUCE_ERR_UNSUPPORTED. */
int reduce_multi(int dtype, int op, const void* in_local, size_t n_local, void* out,
                 reduce_stream_t stream, void* comm);
int reduce_multi_ex(int dtype, int op, const void* in_local, size_t n_local, void* out,
                    reduce_stream_t stream, void* comm, const reduce_opts_t* opts);

int reduce_comm_unique_id_bytes(void);           /* 128 (sizeof ncclUniqueId) */
int reduce_comm_get_unique_id(void* id_out);     /* rank 0; broadcast the bytes */
int reduce_comm_init(void** comm_out, const void* id, int nranks, int rank); /* after cudaSetDevice */
int reduce_comm_destroy(void* comm);
int reduce_comm_count(void* comm, int* nranks);   /* ncclCommCount: ranks in the communicator */

/* ---- sharded mode with the cross-GPU combine fused into the kernel --------
 * (the one-shot combine "fused as the epilogue of the last
 * block").  A team is k ranks (one per GPU, or several on one GPU); each owns a
 * small device buffer that every member maps: across processes through CUDA
 * IPC handles (peer memory over NVLink / NVSwitch), within one process through
 * plain pointers.  reduce_multi_team: every member calls it (same order of
 * calls on every rank) with its local shard; the block that completes a
 * rank's local reduction stores the raw value into every member's buffer
 * (P2P), each 4-byte word paired with the call's epoch in one 8-byte access,
 * polls its own buffer until all k values carry the epoch and combines them
 * in rank order -- no collective launch, no fences, deterministic for a fixed
 * team.  Every member's *out receives the global result.
 *   reduce_team_create(&t, k, rank, handle_out)  handle_out: reduce_team_ipc_handle_bytes() bytes (or NULL)
 *   reduce_team_connect(t, handles)             k handles, rank order, from every member (IPC)
 *   reduce_team_connect_local(t, bufs)          k device pointers (reduce_team_buffer of each member)
 * The call counter (epoch) that sequences the exchange lives in the member's
 * device buffer and is advanced by the kernel, so team calls may be captured
 * into CUDA graphs and replayed (each replay is one call).  A member that
 * never calls leaves the others waiting (as with any collective); after ~2^35
 * cycles (> 15 s) the waiting kernel traps and the caller's sync reports it. */
int reduce_team_create(void** team_out, int nranks, int rank, void* ipc_handle_out);
int reduce_team_ipc_handle_bytes(void);
void* reduce_team_buffer(void* team);
int reduce_team_connect(void* team, const void* handles);
int reduce_team_connect_local(void* team, void* const* bufs);
int reduce_team_destroy(void* team);
int reduce_multi_team(int dtype, int op, const void* in_local, size_t n_local, void* out, reduce_stream_t stream,
                      void* team, const reduce_opts_t* opts);

/* ---- sharded mode with an NVLink SHARP (NVLS) combine -----------------------
 * (SURVEY 8(f) N2 as named there: NCCL symmetric memory + multimem).
 *   reduce_nvls_create(&v, comm, mode): a COLLECTIVE over the NCCL
 *     communicator `comm` (every rank calls it, after cudaSetDevice): each
 *     rank ncclMemAlloc's a 2 MB buffer and registers it as a symmetric window
 *     (ncclCommWindowRegister, NCCL_WIN_COLL_SYMMETRIC); ncclDevCommCreate with
 *     lsaMultimem binds the windows to an NVLS multicast object.  mode 1: the
 *     per-rank values are reduced IN THE NVSWITCH by one multimem.ld_reduce
 *     after a barrier of one multimem.red per rank; mode 2: each rank puts its
 *     value with the call's epoch into every rank's window with one multicast
 *     store (multimem.st) and combines the k values locally in rank order
 *     (deterministic).  Returns REDUCE_ERR_UNSUPPORTED -- with nothing left
 *     allocated -- when the ranks do not share one NVLink domain with
 *     multicast (a single GPU, no NVSwitch, NCCL without NVLS / symmetric
 *     memory); `comm` stays usable for reduce_multi.  Every rank must get the
 *     same status (the calls inside are collectives).
 *   reduce_multi_nvls: as reduce_multi / reduce_multi_team (every rank calls
 *     it with its own shard, in the same order; every rank's *out gets the
 *     global result), the exchange fused into the kernel that completes the
 *     rank's local reduction -- no NCCL launch per call, graph-capturable (the
 *     call counters live in device memory).  REDUCE_MODE_DETERMINISTIC uses
 *     mode 2's rank-order combine whatever `mode` was.
 *   reduce_nvls_destroy: after every rank's last call completed (collective:
 *     window deregistration). */
int reduce_nvls_create(void** nvls_out, void* comm, int mode);
/* The local preconditions of reduce_nvls_create, no collective entered: NCCL
 * with symmetric memory loadable, at least two ranks in `comm`, a multicast-
 * capable device.  Ranks should agree on it (e.g. over their process group)
 * before any of them calls reduce_nvls_create, so that no rank enters the
 * collective registration alone. */
int reduce_nvls_supported(void* comm);
/* A one-member multicast team on the current GPU, built with the CUDA driver's
 * multicast API instead of NCCL (no second GPU needed): the same kernels and
 * protocol at k = 1 -- multimem.st / multimem.red / multimem.ld_reduce through
 * a real multicast object -- for tests and diagnostics.  Use it with
 * reduce_multi_nvls; REDUCE_ERR_UNSUPPORTED where the device has no
 * multicast. */
int reduce_nvls_create_local(void** nvls_out, int mode);
int reduce_nvls_destroy(void* nvls);
int reduce_multi_nvls(int dtype, int op, const void* in_local, size_t n_local, void* out, reduce_stream_t stream,
                      void* nvls, const reduce_opts_t* opts);

/* ---- diagnostics ---------------------------------------------------------- */
const char* reduce_status_string(int status);
const char* reduce_last_error(void);   /* thread-local detail of the last failure */
int reduce_version(void);              /* 10000*major + 100*minor + patch */
void reduce_shutdown(void);            /* free all library-owned workspaces */

#ifdef __cplusplus
}
#endif
#endif /* REDUCE_B200_H */
