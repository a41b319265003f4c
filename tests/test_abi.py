"""Boundary tests that need no GPU: the C-ABI library loads, exports every
function include/reduce.h declares, rejects bad arguments before touching
CUDA, and plans launches (step S0) as DESIGN.md describes."""
import ctypes
import os
import re

import pytest

import paper_conf_cgo_gonzalohghmh19_b200 as rb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "reduce.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?(?:int|void|char)\s*\*?\s*(reduce_\w+|reduce)\s*\(", src, flags=re.M)))


def test_header_symbols_exported():
    names = header_functions()
    assert len(names) >= 17, names
    assert set(names) == set(rb.ABI_SYMBOLS)
    L = ctypes.CDLL(rb.LIB_PATH)
    for name in names:
        assert hasattr(L, name), name


def test_library_is_sm100a_only():
    out = os.popen(f"cuobjdump --list-elf {rb.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out
    assert "sm_90" not in out and "sm_80" not in out


def test_status_strings_and_version():
    assert rb.status_string(0) == "REDUCE_OK"
    assert rb.status_string(6) == "REDUCE_ERR_NOT_PREPARED"
    assert rb.status_string(99) == "REDUCE_ERR_UNKNOWN"
    assert rb.lib.reduce_version() >= 100
    assert rb.lib.reduce_comm_unique_id_bytes() == 128


def _ex(dtype, op, inp, n, out, opts=None):
    return rb.lib.reduce_ex(dtype, op, ctypes.c_void_p(inp), n, ctypes.c_void_p(out), None,
                            ctypes.byref(opts) if opts is not None else None)


@pytest.mark.parametrize("args,why", [
    ((3, 0, 4096, 10, 8192), "bad dtype"),
    ((-1, 0, 4096, 10, 8192), "bad dtype"),
    ((0, 3, 4096, 10, 8192), "bad op"),
    ((0, 0, None, 10, 8192), "NULL in with n > 0"),
    ((0, 0, 4096, 10, None), "NULL out"),
    ((0, 0, 4098, 10, 8192), "misaligned int32 in"),
    ((2, 0, 4100, 10, 8192), "misaligned fp64 in"),
    ((2, 0, 4096, 10, 8196), "misaligned fp64 out"),
])
def test_invalid_arguments_rejected_without_cuda(args, why):
    st = _ex(*args)
    assert st == 1, (why, st, rb.last_error())
    assert rb.last_error()


@pytest.mark.parametrize("kw", [
    dict(mode=7), dict(grid_combine=9), dict(grid_combine=6), dict(block_combine=5), dict(unroll=3),
    dict(block=48), dict(block=2048), dict(block=1024, unroll=8), dict(grid=-2), dict(grid=-5),
    dict(mode="deterministic", grid_combine=rb.GC_ATOMIC),
    dict(mode="deterministic", block_combine=rb.BC_SMEM_ATOMIC_ALL),
    dict(block=96, block_combine=rb.BC_SMEM_TREE),
    dict(stage=3), dict(stage="smem", unroll=2), dict(stage="reg", unroll=16),
    dict(stage="smem", block=1024, unroll=8), dict(grid_combine=4, grid=17),
])
def test_invalid_options_rejected(kw):
    o = rb.make_opts(**kw)
    assert _ex(1, 0, 4096, 1000, 8192, o) == 1, rb.last_error()


def test_query_plan_partition_and_head_tail():
    # fp32, pointer 4 bytes past a 32-byte boundary: 7 head elements
    p = rb.query_plan("float32", "sum", 1000, in_ptr=0x10004)
    assert p["head"] == 7 and p["tail"] == (1000 - 7) % 8
    p = rb.query_plan("float64", "sum", 1000, in_ptr=0x10008)
    assert p["head"] == 3 and p["tail"] == (1000 - 3) % 4
    p = rb.query_plan("int32", "max", 5, in_ptr=0x10004)
    assert p["head"] == 5 and p["tail"] == 0
    p = rb.query_plan("int32", "sum", 0)
    assert p["grid"] == 1 and p["grid_combine"] == rb.GC_DIRECT


def test_query_plan_modes():
    n = 1 << 28
    fast = rb.query_plan("float32", "sum", n, mode="fast")
    det = rb.query_plan("float32", "sum", n, mode="deterministic")
    assert fast["grid_combine"] == rb.GC_ATOMIC and fast["launches"] == 1
    # deterministic: a fixed-order combine (the tuner's pick), never value atomics
    assert det["grid_combine"] in (rb.GC_TWO_PASS, rb.GC_LAST_BLOCK, rb.GC_FLAGS)
    assert det["launches"] == (2 if det["grid_combine"] == rb.GC_TWO_PASS else 1)
    assert det["grid"] <= (1 << 13 if det["grid_combine"] == rb.GC_FLAGS else 1 << 16)
    # one block per 32 KiB tile at the headline size
    tile = fast["block"] * fast["unroll"] * 32
    assert fast["tiles"] == (n * 4) // tile and fast["grid"] == fast["tiles"]
    small = rb.query_plan("float32", "sum", 1000)
    assert small["grid"] == 1 and small["grid_combine"] == rb.GC_DIRECT


def test_query_plan_chain_bounds():
    # chain L: per-thread + lane tree + warp + block + grid terms (S5)
    p = rb.query_plan("float32", "sum", 1 << 28)
    assert 0 < p["chain"] < 64
    p = rb.query_plan("float64", "sum", 1 << 26, mode="deterministic")
    assert p["chain"] < 200
    assert rb.query_plan("int32", "sum", 1 << 20)["chain"] == 0
    assert rb.query_plan("float32", "max", 1 << 20)["chain"] == 0
    va1 = rb.query_plan("float32", "sum", 1 << 20, block_combine=rb.BC_SMEM_ATOMIC_ALL, block=256)
    assert va1["chain"] >= 256


def test_forced_overrides_respected():
    p = rb.query_plan("float32", "sum", 1 << 24, block=128, unroll=8, grid=300,
                      grid_combine=rb.GC_LAST_BLOCK, block_combine=rb.BC_SMEM_TREE)
    assert (p["block"], p["unroll"], p["grid"], p["grid_combine"], p["block_combine"]) == (128, 8, 300, 3, 3)
    assert p["tiles"] == ((1 << 24) // 8 + 128 * 8 - 1) // (128 * 8)


def test_query_plan_staging():
    p = rb.query_plan("float32", "sum", 1 << 28, stage="smem", block=256, unroll=8)
    assert p["stage"] == rb.STAGE_SMEM and p["tiles"] == (1 << 28) // (8 * 256 * 8)
    p = rb.query_plan("float32", "sum", 1 << 28, stage="reg", unroll=4, block=256)
    assert p["stage"] == rb.STAGE_REG
    # fp64 min/max register staging is limited to 512 threads at unroll >= 2, smem staging is not
    assert _ex(2, 2, 4096, 1000, 8192, rb.make_opts(block=1024, unroll=2, stage="reg")) == 1
    assert rb.query_plan("float64", "max", 1 << 20, block=1024, unroll=4, stage="smem")["block"] == 1024


def test_segmented_argument_validation():
    L = rb.lib
    o = rb.make_opts(seg_group=5)
    assert L.reduce_segmented(1, 0, 4096, None, 10, 8192, None, None) == 1        # offsets NULL
    assert L.reduce_segmented(1, 0, 4096, 4096, 10, None, None, None) == 1        # out NULL
    assert L.reduce_segmented(5, 0, 4096, 4096, 10, 8192, None, None) == 1        # dtype
    assert L.reduce_batched(1, 0, 4096, 10, 10, 8192, None, ctypes.byref(o)) == 1  # seg_group 5 needs offsets
    o6 = rb.make_opts(seg_group=6)
    assert L.reduce_segmented(1, 0, 4096, 4096, 10, 8192, None, ctypes.byref(o6)) == 1  # seg_group range
    assert L.reduce_batched(2, 0, 4100, 10, 10, 8192, None, None) == 1            # misaligned fp64
    assert L.reduce_batched(1, 0, None, 10, 0, None, None, None) == 0             # no segments: no-op


def test_histogram_argument_validation():
    L = rb.lib
    assert L.reduce_histogram(2, 4096, 10, 0.0, 1.0, 8, 8192, None) == 1   # fp64 input
    assert L.reduce_histogram(0, 4096, 10, 1.0, 1.0, 8, 8192, None) == 1   # lo == hi
    assert L.reduce_histogram(0, 4096, 10, 0.0, float("inf"), 8, 8192, None) == 1
    assert L.reduce_histogram(0, 4096, 10, 0.0, 1.0, 0, 8192, None) == 1   # nbins
    assert L.reduce_histogram(0, 4096, 10, 0.0, 1.0, 8, None, None) == 1   # counts NULL
    assert L.reduce_histogram(0, 4098, 10, 0.0, 1.0, 8, 8192, None) == 1   # misaligned
    assert L.reduce_histogram(0, 4096, 10, 0.5, 10.0, 8, 8192, None) == 1  # int32 needs integer bounds


def test_forced_shape_ignores_table_grid_cap():
    n = 1 << 24
    free = rb.query_plan("float32", "sum", n, block=256, unroll=2, grid_combine=2)
    assert free["grid"] == free["tiles"] == n // (256 * 2 * 8)
    assert rb.query_plan("float32", "sum", n, grid=-1)["grid"] == rb.query_plan("float32", "sum", n, grid=-1)["tiles"]
    assert rb.query_plan("float32", "sum", n, block=256, unroll=2, grid=300)["grid"] == 300


def test_mode_default_roundtrip():
    old = rb.get_mode()
    rb.set_mode("deterministic")
    assert rb.get_mode() == 1
    rb.set_mode(42)  # ignored
    assert rb.get_mode() == 1
    rb.set_mode(old)


def test_shard_range_partitions_exactly():
    for n in (0, 1, 7, 1000, 2 ** 31):
        for k in (1, 2, 3, 8):
            ranges = [rb.shard_range(n, k, r) for r in range(k)]
            assert ranges[0][0] == 0 and ranges[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
            assert max(h - l for l, h in ranges) - min(h - l for l, h in ranges) <= 1


def test_nvls_entry_points_reject_bad_arguments_without_cuda():
    h = ctypes.c_void_p()
    assert rb.lib.reduce_nvls_create_local(ctypes.byref(h), 3) == 1      # bad mode
    assert rb.lib.reduce_nvls_create(ctypes.byref(h), None, 1) == 1      # no communicator
    assert rb.lib.reduce_nvls_create(None, ctypes.c_void_p(8), 1) == 1   # no output
    assert rb.lib.reduce_nvls_destroy(None) == 1
    assert rb.lib.reduce_nvls_supported(None) == 1
    assert rb.lib.reduce_multi_nvls(1, 0, None, 0, None, None, None, None) == 1  # out NULL
    assert "mode" in rb.last_error() or "NULL" in rb.last_error()


def test_binding_rejects_host_tensors_and_bad_outputs_without_cuda():
    """The Python binding validates before any CUDA call: host
    inputs are refused, and caller-supplied outputs are checked (dtype, size,
    device) so the C side never writes past a wrong buffer."""
    import torch
    with pytest.raises(ValueError):
        rb.reduce(torch.ones(4), "sum")
    with pytest.raises(ValueError):
        rb.reduce_segmented(torch.ones(4), torch.zeros(2, dtype=torch.int64), "sum")
    with pytest.raises(ValueError):
        rb.reduce_batched(torch.ones(2, 2), "sum")
    with pytest.raises(ValueError):
        rb.histogram(torch.ones(4), 0.0, 1.0, 4)
    # the output check itself (device-independent parts)
    x = torch.ones(4)
    with pytest.raises(ValueError, match="dtype"):
        rb._check_out(torch.ones(1, dtype=torch.float64), x, 1)
    with pytest.raises(ValueError):
        rb._check_out(torch.ones(1), x, 1)        # not a CUDA tensor
    assert rb._opts_for({}) is None
    o1 = rb._opts_for({"mode": "deterministic", "grid": 8})
    assert rb._opts_for({"grid": 8, "mode": "deterministic"}) is o1 and o1.mode == 1 and o1.grid == 8
    assert rb.make_opts(input_ready=True).flags == rb.FLAG_INPUT_READY


def test_grid_combine_names_cover_every_combine():
    """bench.py labels plans with GC_NAMES: every value the C side accepts has one."""
    assert len(rb.GC_NAMES) == rb.GC_FLAGS + 1 and rb.GC_NAMES[rb.GC_FLAGS] == "flags"
    for gc in range(len(rb.GC_NAMES)):
        p = rb.query_plan("float32", "sum", 1 << 20, grid_combine=gc, **({"grid": 16} if gc == rb.GC_CLUSTER else {}))
        assert p["grid_combine"] == gc
    with pytest.raises(rb.ReduceError):
        rb.query_plan("float32", "sum", 1 << 20, grid_combine=len(rb.GC_NAMES))
