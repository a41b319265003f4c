"""Python binding of libreduce_b200.so (include/reduce.h) — argument marshalling only.

Every step of the reduction runs in the library's sm_100a kernels; this module
only converts tensors / arrays to (pointer, count, dtype) and calls the C ABI
with the same names.  There is no CPU fallback: if the shared library is
missing, importing the binding raises.  (The CPU oracle under ``oracle/`` is
test infrastructure and is never imported here.)

PyTorch is used only for device memory, streams and process groups.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libreduce_b200.so")

INT32, FLOAT32, FLOAT64 = 0, 1, 2
SUM, MIN, MAX, SUM_ACCURATE = 0, 1, 2, 3
MODE_FAST, MODE_DETERMINISTIC = 0, 1
BC_SHFL, BC_SMEM_ATOMIC_WARP, BC_SMEM_ATOMIC_ALL, BC_SMEM_TREE = 0, 1, 2, 3
GC_DIRECT, GC_ATOMIC, GC_TWO_PASS, GC_LAST_BLOCK, GC_CLUSTER, GC_FLAGS = 0, 1, 2, 3, 4, 5
GC_NAMES = ("direct", "atomic", "two_pass", "last_block", "cluster", "flags")  # indexed by reduce_grid_combine_t
STAGE_REG, STAGE_SMEM = 1, 2
FLAG_INPUT_READY = 1
OK = 0

OPS = {"sum": SUM, "min": MIN, "max": MAX, "sum_accurate": SUM_ACCURATE}
DTYPE_NAMES = {"int32": INT32, "float32": FLOAT32, "float64": FLOAT64}
ELEM_BYTES = {INT32: 4, FLOAT32: 4, FLOAT64: 8}

# every symbol include/reduce.h declares (checked by tests/test_abi.py)
ABI_SYMBOLS = (
    "reduce", "reduce_ex", "reduce_query_plan", "reduce_prepare", "reduce_set_mode",
    "reduce_get_mode", "reduce_host", "reduce_multi", "reduce_multi_ex",
    "reduce_comm_unique_id_bytes", "reduce_comm_get_unique_id", "reduce_comm_init",
    "reduce_comm_destroy", "reduce_comm_count", "reduce_status_string", "reduce_last_error", "reduce_version",
    "reduce_shutdown", "reduce_segmented", "reduce_batched", "reduce_histogram",
    "reduce_team_create", "reduce_team_ipc_handle_bytes", "reduce_team_buffer", "reduce_team_connect",
    "reduce_team_connect_local", "reduce_team_destroy", "reduce_multi_team",
    "reduce_nvls_create", "reduce_nvls_create_local", "reduce_nvls_supported", "reduce_nvls_destroy",
    "reduce_multi_nvls",
)


class ReduceError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = f"{where}: {status_string(status)}: {last_error()}"
        super().__init__(msg)


class reduce_opts_t(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int), ("grid_combine", ctypes.c_int), ("block_combine", ctypes.c_int),
                ("block", ctypes.c_int), ("unroll", ctypes.c_int), ("grid", ctypes.c_int),
                ("seg_group", ctypes.c_int), ("stage", ctypes.c_int), ("flags", ctypes.c_int)]


class reduce_plan_t(ctypes.Structure):
    _fields_ = [("grid_combine", ctypes.c_int), ("block_combine", ctypes.c_int),
                ("grid", ctypes.c_int), ("block", ctypes.c_int), ("unroll", ctypes.c_int),
                ("stage", ctypes.c_int), ("launches", ctypes.c_int), ("slots", ctypes.c_int),
                ("head", ctypes.c_int), ("tail", ctypes.c_int),
                ("tiles", ctypes.c_longlong), ("chain", ctypes.c_longlong)]

    def as_dict(self) -> dict:
        return {f: getattr(self, f) for f, _ in self._fields_}


def _load() -> ctypes.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
            "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
    vp, sz, i = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int
    opts_p, plan_p = ctypes.POINTER(reduce_opts_t), ctypes.POINTER(reduce_plan_t)
    sigs = {
        "reduce": (i, [i, i, vp, sz, vp, vp]),
        "reduce_ex": (i, [i, i, vp, sz, vp, vp, opts_p]),
        "reduce_query_plan": (i, [i, i, vp, sz, opts_p, plan_p]),
        "reduce_prepare": (i, [vp, sz]),
        "reduce_set_mode": (None, [i]),
        "reduce_get_mode": (i, []),
        "reduce_host": (i, [i, i, vp, sz, vp, vp, opts_p]),
        "reduce_multi": (i, [i, i, vp, sz, vp, vp, vp]),
        "reduce_multi_ex": (i, [i, i, vp, sz, vp, vp, vp, opts_p]),
        "reduce_comm_unique_id_bytes": (i, []),
        "reduce_comm_get_unique_id": (i, [vp]),
        "reduce_comm_init": (i, [ctypes.POINTER(vp), vp, i, i]),
        "reduce_comm_destroy": (i, [vp]),
        "reduce_comm_count": (i, [vp, ctypes.POINTER(i)]),
        "reduce_status_string": (ctypes.c_char_p, [i]),
        "reduce_last_error": (ctypes.c_char_p, []),
        "reduce_version": (i, []),
        "reduce_shutdown": (None, []),
        "reduce_segmented": (i, [i, i, vp, vp, sz, vp, vp, opts_p]),
        "reduce_batched": (i, [i, i, vp, sz, sz, vp, vp, opts_p]),
        "reduce_histogram": (i, [i, vp, sz, ctypes.c_double, ctypes.c_double, i, vp, vp]),
        "reduce_team_create": (i, [ctypes.POINTER(vp), i, i, vp]),
        "reduce_team_ipc_handle_bytes": (i, []),
        "reduce_team_buffer": (vp, [vp]),
        "reduce_team_connect": (i, [vp, vp]),
        "reduce_team_connect_local": (i, [vp, ctypes.POINTER(vp)]),
        "reduce_team_destroy": (i, [vp]),
        "reduce_multi_team": (i, [i, i, vp, sz, vp, vp, vp, opts_p]),
        "reduce_nvls_create": (i, [ctypes.POINTER(vp), vp, i]),
        "reduce_nvls_create_local": (i, [ctypes.POINTER(vp), i]),
        "reduce_nvls_supported": (i, [vp]),
        "reduce_nvls_destroy": (i, [vp]),
        "reduce_multi_nvls": (i, [i, i, vp, sz, vp, vp, vp, opts_p]),
    }
    for name, (res, args) in sigs.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


lib = _load()


def status_string(status: int) -> str:
    return lib.reduce_status_string(status).decode()


def last_error() -> str:
    return lib.reduce_last_error().decode()


def _check(status: int, where: str) -> None:
    if status != OK:
        raise ReduceError(status, where)


def make_opts(mode=None, grid_combine=None, block_combine=None, block=0, unroll=0, grid=0, stage=0, seg_group=0,
              input_ready=False, flags=0):
    """reduce_opts_t from keywords.  input_ready=True sets REDUCE_FLAG_INPUT_READY
    (the caller guarantees no kernel still running writes the input: early loads
    allowed, include/reduce.h "Stream ordering")."""
    if isinstance(mode, str):
        mode = {"fast": MODE_FAST, "deterministic": MODE_DETERMINISTIC}[mode]
    if isinstance(stage, str):
        stage = {"auto": 0, "reg": STAGE_REG, "smem": STAGE_SMEM}[stage]
    return reduce_opts_t(-1 if mode is None else int(mode),
                         -1 if grid_combine is None else int(grid_combine),
                         -1 if block_combine is None else int(block_combine),
                         int(block), int(unroll), int(grid), int(seg_group), int(stage),
                         int(flags) | (FLAG_INPUT_READY if input_ready else 0))


def _op(op) -> int:
    return OPS[op] if isinstance(op, str) else int(op)


_TORCH_DT = {}


def _torch_dtype_code(t) -> int:
    if not _TORCH_DT:
        import torch
        _TORCH_DT.update({torch.int32: INT32, torch.float32: FLOAT32, torch.float64: FLOAT64})
    code = _TORCH_DT.get(t.dtype)
    if code is None:
        raise TypeError(f"unsupported dtype {t.dtype} (int32, float32, float64)")
    return code


def _stream_handle(stream, device=None) -> int:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream(device)
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _check_cuda_in(x, what: str = "input") -> None:
    if not x.is_cuda:
        raise ValueError(f"{what} must be a CUDA tensor")
    if not x.is_contiguous():
        raise ValueError(f"{what} must be contiguous")


def _check_out(out, x, count: int, dtype=None) -> None:
    """A caller-supplied output must hold `count` elements of the result dtype,
    contiguous, on x's device (the C side writes count * sizeof(T) bytes)."""
    want = x.dtype if dtype is None else dtype
    if out.dtype != want:
        raise ValueError(f"out has dtype {out.dtype}, expected {want}")
    if not out.is_cuda or out.device != x.device:
        raise ValueError(f"out must be a CUDA tensor on {x.device}, got {out.device}")
    if not out.is_contiguous():
        raise ValueError("out must be contiguous")
    if out.numel() < count:
        raise ValueError(f"out holds {out.numel()} elements, needs {count}")


class _on_device:
    """Make x's device current for the C call (the library resolves its
    workspace and launches on the current device; the stream comes from x)."""

    def __init__(self, dev):
        self.dev = dev

    def __enter__(self):
        import torch
        self.prev = torch.cuda.current_device()
        if self.dev.index is not None and self.dev.index != self.prev:
            torch.cuda.set_device(self.dev)
        return self

    def __exit__(self, *a):
        import torch
        if torch.cuda.current_device() != self.prev:
            torch.cuda.set_device(self.prev)


def reduce_ptr(dtype: int, op, in_ptr: int, n: int, out_ptr: int, stream: int = 0, opts=None) -> None:
    """Raw-pointer form of reduce_ex (device pointers, stream handle)."""
    st = lib.reduce_ex(dtype, OPS[op] if op.__class__ is str else op, in_ptr or None, n, out_ptr or None,
                       stream or None, None if opts is None else ctypes.byref(opts))
    if st:
        raise ReduceError(st, "reduce_ex")


_OPTS_CACHE: dict = {}


def _opts_for(opt_kw):
    """reduce_opts_t for keyword options, cached (the C side copies it per call)."""
    if not opt_kw:
        return None
    key = tuple(sorted(opt_kw.items()))
    o = _OPTS_CACHE.get(key)
    if o is None:
        o = make_opts(**opt_kw)
        if len(_OPTS_CACHE) < 4096:
            _OPTS_CACHE[key] = o
    return o


def reduce(x, op="sum", out=None, stream=None, **opt_kw):
    """Reduce a contiguous CUDA tensor to a 1-element device tensor (async)."""
    dev = x.get_device()  # -1 for host tensors
    if dev < 0:
        raise ValueError("reduce() takes a CUDA tensor; use reduce_host() for host data")
    if not x.is_contiguous():
        raise ValueError("input must be contiguous")
    dt = _torch_dtype_code(x)
    if out is None:
        import torch
        out = torch.empty(1, dtype=x.dtype, device=x.device)
    elif out.dtype is not x.dtype or out.get_device() != dev or not out.is_contiguous() or out.numel() < 1:
        _check_out(out, x, 1)  # raises with the reason
    opts = _opts_for(opt_kw)
    s = stream.cuda_stream if stream is not None and not isinstance(stream, int) else _stream_handle(stream, x.device)
    import torch
    if torch.cuda.current_device() == dev:
        reduce_ptr(dt, op, x.data_ptr(), x.numel(), out.data_ptr(), s, opts)
    else:
        with torch.cuda.device(dev):
            reduce_ptr(dt, op, x.data_ptr(), x.numel(), out.data_ptr(), s, opts)
    return out


def reduce_segmented(x, offsets, op="sum", out=None, stream=None, **opt_kw):
    """out[i] = reduce(x[offsets[i]:offsets[i+1]]) for a CUDA tensor x and a CUDA
    int64 tensor offsets of num_segments + 1 entries (one launch, deterministic)."""
    import torch
    dt = _torch_dtype_code(x)
    _check_cuda_in(x)
    nseg = offsets.numel() - 1
    if offsets.dtype != torch.int64 or not offsets.is_cuda or not offsets.is_contiguous():
        raise ValueError("offsets must be a contiguous CUDA int64 tensor")
    if offsets.device != x.device:
        raise ValueError("offsets must be on the input's device")
    if out is None:
        out = torch.empty(max(nseg, 0), dtype=x.dtype, device=x.device)
    else:
        _check_out(out, x, max(nseg, 0))
    opts = make_opts(**opt_kw) if opt_kw else None
    with _on_device(x.device):
        st = lib.reduce_segmented(dt, _op(op), x.data_ptr() or None, offsets.data_ptr() or None, max(nseg, 0),
                                  out.data_ptr() or None, _stream_handle(stream, x.device),
                                  ctypes.byref(opts) if opts is not None else None)
    _check(st, "reduce_segmented")
    return out


def reduce_batched(x, op="sum", out=None, stream=None, **opt_kw):
    """Row reductions of a contiguous 2-D CUDA tensor (rows x seg_len) in one launch."""
    import torch
    dt = _torch_dtype_code(x)
    if x.dim() != 2 or not x.is_contiguous():
        raise ValueError("reduce_batched takes a contiguous 2-D tensor")
    _check_cuda_in(x)
    rows, cols = x.shape
    if out is None:
        out = torch.empty(rows, dtype=x.dtype, device=x.device)
    else:
        _check_out(out, x, rows)
    opts = make_opts(**opt_kw) if opt_kw else None
    with _on_device(x.device):
        st = lib.reduce_batched(dt, _op(op), x.data_ptr() or None, cols, rows, out.data_ptr() or None,
                                _stream_handle(stream, x.device), ctypes.byref(opts) if opts is not None else None)
    _check(st, "reduce_batched")
    return out


def histogram(x, lo: float, hi: float, nbins: int, counts=None, stream=None):
    """counts[b] = #{lo <= x < hi, b = floor((x - lo) * nbins / (hi - lo))} (CUDA int32/fp32 tensor)."""
    import torch
    dt = _torch_dtype_code(x)
    _check_cuda_in(x)
    if counts is None:
        counts = torch.empty(nbins, dtype=torch.int32, device=x.device)  # bit pattern of uint32 counts
    else:
        _check_out(counts, x, int(nbins), dtype=torch.int32)
    with _on_device(x.device):
        st = lib.reduce_histogram(dt, x.data_ptr() or None, x.numel(), float(lo), float(hi), int(nbins),
                                  counts.data_ptr(), _stream_handle(stream, x.device))
    _check(st, "reduce_histogram")
    return counts


def query_plan(dtype, op, n: int, in_ptr: int = 0, **opt_kw) -> dict:
    dt = DTYPE_NAMES[dtype] if isinstance(dtype, str) else int(dtype)
    plan = reduce_plan_t()
    opts = make_opts(**opt_kw) if opt_kw else None
    st = lib.reduce_query_plan(dt, _op(op), ctypes.c_void_p(in_ptr or None), n,
                               ctypes.byref(opts) if opts is not None else None, ctypes.byref(plan))
    _check(st, "reduce_query_plan")
    return plan.as_dict()


def prepare(stream=None, max_n: int = 0) -> None:
    _check(lib.reduce_prepare(ctypes.c_void_p(_stream_handle(stream)), max_n), "reduce_prepare")


def set_mode(mode) -> None:
    if isinstance(mode, str):
        mode = {"fast": MODE_FAST, "deterministic": MODE_DETERMINISTIC}[mode]
    lib.reduce_set_mode(int(mode))


def get_mode() -> int:
    return lib.reduce_get_mode()


def reduce_host(x, op="sum", stream=None, **opt_kw):
    """End-to-end: host array/tensor in, Python scalar out (copies inside the call)."""
    import numpy as np
    if hasattr(x, "numpy") and not isinstance(x, np.ndarray):
        if x.is_cuda:
            raise ValueError("reduce_host() takes host memory")
        dt = _torch_dtype_code(x)
        ptr, n = x.data_ptr(), x.numel()
        npdt = {INT32: np.int32, FLOAT32: np.float32, FLOAT64: np.float64}[dt]
    else:
        x = np.ascontiguousarray(x)
        npdt = x.dtype.type
        dt = {np.dtype(np.int32): INT32, np.dtype(np.float32): FLOAT32, np.dtype(np.float64): FLOAT64}[x.dtype]
        ptr, n = x.ctypes.data, x.size
    res = np.zeros(1, dtype=npdt)
    opts = make_opts(**opt_kw) if opt_kw else None
    st = lib.reduce_host(dt, _op(op), ctypes.c_void_p(ptr or None), n, ctypes.c_void_p(res.ctypes.data),
                         ctypes.c_void_p(_stream_handle(stream)), ctypes.byref(opts) if opts is not None else None)
    _check(st, "reduce_host")
    return res[0]


# ------------------------------------------------------------- sharded mode
def broadcast_unique_id(group=None) -> bytes:
    """Rank 0 of `group` creates an NCCL unique id (reduce_comm_get_unique_id);
    it is broadcast to every rank through the torch process group (any backend)."""
    import torch.distributed as dist
    rank = dist.get_rank(group)
    nbytes = lib.reduce_comm_unique_id_bytes()
    obj = [None]
    if rank == 0:
        uid = (ctypes.c_char * nbytes)()
        _check(lib.reduce_comm_get_unique_id(ctypes.cast(uid, ctypes.c_void_p)), "reduce_comm_get_unique_id")
        obj = [bytes(uid)]
    src = dist.get_global_rank(group, 0) if group is not None else 0
    dist.broadcast_object_list(obj, src=src, group=group)
    if not isinstance(obj[0], bytes) or len(obj[0]) != nbytes:
        raise RuntimeError("bad NCCL unique id received")
    return obj[0]


class Comm:
    """An NCCL communicator owned by the library (reduce_comm_init), bootstrapped
    over a torch.distributed process group (the unique id travels through it).
    Call after torch.cuda.set_device(local_rank)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        uid_bytes = broadcast_unique_id(group)
        uid = (ctypes.c_char * len(uid_bytes)).from_buffer_copy(uid_bytes)
        handle = ctypes.c_void_p()
        _check(lib.reduce_comm_init(ctypes.byref(handle), ctypes.cast(uid, ctypes.c_void_p), world, rank),
               "reduce_comm_init")
        self.handle = handle.value
        self.rank, self.world = rank, world

    def nranks(self) -> int:
        """ncclCommCount of the communicator (ranks NCCL itself sees)."""
        k = ctypes.c_int(0)
        _check(lib.reduce_comm_count(ctypes.c_void_p(self.handle), ctypes.byref(k)), "reduce_comm_count")
        return k.value

    def destroy(self) -> None:
        if self.handle:
            _check(lib.reduce_comm_destroy(ctypes.c_void_p(self.handle)), "reduce_comm_destroy")
            self.handle = None


def reduce_multi(x, op, comm: Comm, out=None, stream=None, **opt_kw):
    """Every rank passes its local CUDA shard; every rank gets the global result."""
    import torch
    dt = _torch_dtype_code(x)
    _check_cuda_in(x)
    if out is None:
        out = torch.empty(1, dtype=x.dtype, device=x.device)
    else:
        _check_out(out, x, 1)
    opts = make_opts(**opt_kw) if opt_kw else None
    st = lib.reduce_multi_ex(dt, _op(op), ctypes.c_void_p(x.data_ptr() or None), x.numel(),
                             ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(_stream_handle(stream, x.device)),
                             ctypes.c_void_p(comm.handle), ctypes.byref(opts) if opts is not None else None)
    _check(st, "reduce_multi_ex")
    return out


class Team:
    """Ranks whose per-rank results meet through peer memory inside the kernel
    (reduce_multi_team).  Team(group) exchanges CUDA IPC handles
    over a torch.distributed group (one process per GPU, or several processes on
    one GPU); Team.local(k) makes k in-process members (e.g. one per stream)."""

    def __init__(self, group=None, _local=None):
        if _local is not None:
            self.handle, self.rank, self.world = _local
            return
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        nb = lib.reduce_team_ipc_handle_bytes()
        hbuf = (ctypes.c_char * nb)()
        handle = ctypes.c_void_p()
        # every step is agreed over the group, so a failure on one rank raises on
        # all of them instead of leaving the others blocked in a collective
        st = lib.reduce_team_create(ctypes.byref(handle), world, rank, ctypes.cast(hbuf, ctypes.c_void_p))
        err = None if st == OK else (st, last_error())
        allh = [None] * world
        dist.all_gather_object(allh, (st, bytes(hbuf)), group=group)
        if st == OK and all(s == OK for s, _ in allh):
            joined = (ctypes.c_char * (nb * world)).from_buffer_copy(b"".join(h for _, h in allh))
            st = lib.reduce_team_connect(handle, ctypes.cast(joined, ctypes.c_void_p))
            err = None if st == OK else (st, last_error())
        else:
            st = st if st != OK else next(s for s, _ in allh if s != OK)
        sts = [None] * world
        dist.all_gather_object(sts, st, group=group)
        if any(s != OK for s in sts):
            if handle.value:
                lib.reduce_team_destroy(handle)
            bad = next(r for r, s in enumerate(sts) if s != OK)
            raise ReduceError(sts[bad], f"Team (rank {bad} failed{'' if err is None else ': ' + err[1]})")
        self.handle, self.rank, self.world = handle.value, rank, world

    @classmethod
    def local(cls, k: int):
        hs = []
        for r in range(k):
            h = ctypes.c_void_p()
            _check(lib.reduce_team_create(ctypes.byref(h), k, r, None), "reduce_team_create")
            hs.append(h.value)
        bufs = (ctypes.c_void_p * k)(*[lib.reduce_team_buffer(h) for h in hs])
        for h in hs:
            _check(lib.reduce_team_connect_local(h, bufs), "reduce_team_connect_local")
        return [cls(_local=(h, r, k)) for r, h in enumerate(hs)]

    def destroy(self) -> None:
        if self.handle:
            _check(lib.reduce_team_destroy(self.handle), "reduce_team_destroy")
            self.handle = None


def reduce_multi_team(x, op, team: Team, out=None, stream=None, **opt_kw):
    """Every team member passes its local CUDA shard; every member gets the global result."""
    import torch
    dt = _torch_dtype_code(x)
    _check_cuda_in(x)
    if out is None:
        out = torch.empty(1, dtype=x.dtype, device=x.device)
    else:
        _check_out(out, x, 1)
    opts = make_opts(**opt_kw) if opt_kw else None
    st = lib.reduce_multi_team(dt, _op(op), x.data_ptr() or None, x.numel(), out.data_ptr(),
                               _stream_handle(stream, x.device), team.handle,
                               ctypes.byref(opts) if opts is not None else None)
    _check(st, "reduce_multi_team")
    return out


class Nvls:
    """The NVLink SHARP (multicast) combine of reduce_multi_nvls, built over an
    NCCL communicator (a Comm) -- a collective: every rank constructs it.
    mode 1: in-switch multimem.ld_reduce; mode 2: multicast store + rank-order
    combine.  Raises ReduceError(REDUCE_ERR_UNSUPPORTED) on every rank when the
    ranks have no NVLS multicast (e.g. one GPU)."""

    UNSUPPORTED = 2

    def __init__(self, comm: "Comm" = None, mode: int = 1, group=None, _local=None):
        if _local is not None:
            self.handle, self.rank, self.world, self.mode = _local, 0, 1, mode
            return
        import torch.distributed as dist
        world = comm.world

        def agree(st, err):
            sts = [None] * world
            if dist.is_initialized():
                dist.all_gather_object(sts, (st, err), group=group)
            else:
                sts = [(st, err)]
            return sts
        # the local preconditions first, agreed by every rank: nobody enters the
        # collective registration alone
        st = lib.reduce_nvls_supported(ctypes.c_void_p(comm.handle))
        sts = agree(st, last_error() if st != OK else "")
        h = ctypes.c_void_p()
        if all(s == OK for s, _ in sts):
            st = lib.reduce_nvls_create(ctypes.byref(h), ctypes.c_void_p(comm.handle), int(mode))
            sts = agree(st, last_error() if st != OK else "")
        if any(s != OK for s, _ in sts):
            if st == OK and h.value:
                lib.reduce_nvls_destroy(h)
            bad = next(r for r, (s, _) in enumerate(sts) if s != OK)
            raise ReduceError(sts[bad][0], f"Nvls (rank {bad}: {sts[bad][1]})")
        self.handle, self.rank, self.world, self.mode = h.value, comm.rank, world, mode

    @classmethod
    def local(cls, mode: int = 1) -> "Nvls":
        """One-member multicast team on the current GPU (driver multicast API,
        no NCCL): the NVLS kernels at k = 1, for tests on a single GPU."""
        h = ctypes.c_void_p()
        _check(lib.reduce_nvls_create_local(ctypes.byref(h), int(mode)), "reduce_nvls_create_local")
        return cls(_local=h.value, mode=mode)

    def destroy(self) -> None:
        if self.handle:
            _check(lib.reduce_nvls_destroy(ctypes.c_void_p(self.handle)), "reduce_nvls_destroy")
            self.handle = None


def reduce_multi_nvls(x, op, nvls: Nvls, out=None, stream=None, **opt_kw):
    """Every rank passes its local CUDA shard; every rank gets the global result
    (cross-GPU combine through NVLS multicast inside the reduction kernel)."""
    import torch
    dt = _torch_dtype_code(x)
    _check_cuda_in(x)
    if out is None:
        out = torch.empty(1, dtype=x.dtype, device=x.device)
    else:
        _check_out(out, x, 1)
    opts = make_opts(**opt_kw) if opt_kw else None
    st = lib.reduce_multi_nvls(dt, _op(op), x.data_ptr() or None, x.numel(), out.data_ptr(),
                               _stream_handle(stream, x.device), nvls.handle,
                               ctypes.byref(opts) if opts is not None else None)
    _check(st, "reduce_multi_nvls")
    return out


def shard_range(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous shard [lo, hi) of rank r: floor(r*n/k) .. floor((r+1)*n/k)."""
    return (rank * n) // world, ((rank + 1) * n) // world
