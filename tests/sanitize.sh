#!/usr/bin/env bash
# compute-sanitizer pass over every kernel family (SURVEY section 4 "Sanitizers"):
# memcheck, racecheck, synccheck and initcheck on small ragged sizes, every grid
# combine (DIRECT, ATOMIC, TWO_PASS, LAST_BLOCK, CLUSTER, FLAGS), both staging modes,
# every segmented group with and without the long-segment queue, the histogram
# bin-replication and quotient paths, and the team combine.
# Usage (GPU box): bash tests/sanitize.sh  -> exit 0 iff every tool reports 0 errors.
set -u
cd "$(dirname "$0")/.."
CS=${CS:-/usr/local/cuda/bin/compute-sanitizer}
cat > /tmp/rb_sanitize_case.py <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_cgo_gonzalohghmh19_b200 as rb
for dt in (torch.int32, torch.float32, torch.float64):
    for n in (1, 33, 4097, (1 << 20) + 3):
        x = torch.arange(n + 3, device="cuda").to(dt)[3:]
        for op in ("sum", "min", "max"):
            for kw in (dict(), dict(mode="deterministic"), dict(grid_combine=3), dict(grid_combine=4, grid=8),
                       dict(stage="smem", unroll=8, block=256), dict(block_combine=1), dict(block_combine=3, block=128),
                       dict(input_ready=True), dict(grid_combine=1, block=32, unroll=1), dict(grid_combine=5),
                       dict(grid_combine=5, block=32, unroll=1), dict(grid_combine=5, mode="deterministic", grid=3)):
                rb.reduce(x, op, **kw)
        if dt != torch.int32:
            rb.reduce(x, "sum_accurate")
            rb.reduce(x, "sum_accurate", mode="deterministic")
    offs = torch.tensor([0, 0, 1, 33, 100, 4097], dtype=torch.int64, device="cuda")
    base = torch.arange(5000, device="cuda").to(dt)[1:]
    # long segments (queued: k_seg_chunks / k_seg_finish) among short ones,
    # a decreasing pair, and few long uniform rows (queued too)
    loffs = torch.tensor([0, 5, 70005, 70006, 60000, 150003, 150040], dtype=torch.int64, device="cuda")
    lbase = torch.arange(150050, device="cuda").to(dt)[3:]
    # element-balanced path (seg_group 0 / 5): monotone offsets with segments
    # crossing lanes, chunks and warp ranges, a run of 3000 empty segments (the
    # per-piece walk) and a window not starting at element 0
    rng = np.random.Generator(np.random.PCG64(3))
    lens = np.minimum((rng.pareto(1.2, 6000) * 8).astype(np.int64) + 1, 60000)
    lens[2000:5000] = 0
    moffs = torch.from_numpy(np.concatenate([[7], 7 + np.cumsum(lens)])).to("cuda")
    mbase = torch.arange(int(moffs[-1]) + 16, device="cuda").to(dt)[1:]
    for op in ("sum", "min", "max") + (("sum_accurate",) if dt != torch.int32 else ()):
        rb.reduce_segmented(mbase, moffs, op, seg_group=5)
    # aligned short uniform rows (k_rows_aligned: 1, 2, 4 vectors per row and a runtime count)
    abase = torch.arange(8 * 4099, device="cuda").to(dt)
    ve = 4 if dt == torch.float64 else 8
    for nvv in (1, 2, 3, 4, 8):
        rows = abase.numel() // (nvv * ve)
        rb.reduce_batched(abase[: rows * nvv * ve].view(rows, nvv * ve), "max")
        if dt != torch.int32:
            rb.reduce_batched(abase[: rows * nvv * ve].view(rows, nvv * ve), "sum_accurate")
    # tiled rows (k_rows_tiled: 1 KB and 32 KB rows, partial last tile;
    # k_rows_tiled_big: 2048 rows of 64 KB)
    tbase = torch.arange(2048 * 64 * 1024 // 4 + 64, device="cuda").to(dt)[:2048 * 64 * 1024 // dt.itemsize]
    for kb, rows in ((1, 33), (32, 3)):
        cols = kb * 1024 // dt.itemsize
        for op in ("sum", "max") + (("sum_accurate",) if dt != torch.int32 else ()):
            rb.reduce_batched(tbase[:rows * cols].view(rows, cols), op, seg_group=6)
    rb.reduce_batched(tbase.view(2048, -1), "min", seg_group=6)
    if dt != torch.int32:
        rb.reduce_batched(tbase.view(2048, -1), "sum_accurate", seg_group=6)
    for g in (0, 1, 2, 3, 4):
        rb.reduce_segmented(base, offs, "sum", seg_group=g)
        rb.reduce_batched(base[:4096].view(64, 64), "max", seg_group=g)
        rb.reduce_segmented(lbase, loffs, "sum", seg_group=g)
        rb.reduce_batched(lbase[:3 * 40001].view(3, 40001), "min", seg_group=g)
        if dt != torch.int32:
            rb.reduce_segmented(lbase, loffs, "sum_accurate", seg_group=g)
    if dt != torch.float64:
        for nb in (1, 7, 16, 256, 4096, 20000, 20001, 65536, 1 << 20):
            rb.histogram(base, 0, 4000, nb)
        if dt == torch.int32:  # both int32 quotient paths and clamped bounds
            rb.histogram(base, -2.0 ** 31, 2.0 ** 31, 1000)
            rb.histogram(base, 2.0 ** 31 - 10, 2.0 ** 31 + 10, 4)
            rb.histogram(base, 5, 6, 3)
        if dt == torch.int32:
            rb.histogram(base, -2.0 ** 31, 2.0 ** 31, 1000)  # 64-bit quotient path
# team combine (k = 1: members on one GPU cannot run concurrently under the
# sanitizer, which serialises kernels, so k > 1 would wait for itself)
team = rb.Team.local(1)[0]
for dt in (torch.int32, torch.float32, torch.float64):
    for n in (0, 33, (1 << 20) + 3):
        x = torch.arange(n + 1, device="cuda").to(dt)[1:]
        for op in ("sum", "min", "max"):
            for kw in (dict(), dict(mode="deterministic"), dict(grid_combine=4, grid=8), dict(grid_combine=5)):
                rb.reduce_multi_team(x, op, team, **kw)
torch.cuda.synchronize()
team.destroy()
print("ok")
PY
rc=0
for tool in memcheck racecheck synccheck initcheck; do
  extra=""; [ $tool = racecheck ] && extra="--racecheck-report all"
  out=$($CS --tool $tool $extra --error-exitcode 9 python /tmp/rb_sanitize_case.py 2>&1)
  code=$?
  echo "== $tool: exit $code; $(echo "$out" | grep -E 'ERROR SUMMARY|^ok' | tr '\n' ' ')"
  [ $code -ne 0 ] && { echo "$out" | tail -30; rc=1; }
done
exit $rc
