"""A/B: reduce_batched on 256 MB of uniform rows of 1-32 KB -- the tiled-rows
kernel (seg_group 6) against the group kernel the auto choice used before it
(one thread <= 512 B, 8 lanes <= 4 KB, one warp <= 16 KB, one block above; rows of >= 64 KB:
one block per row, k_rows_tiled_big, needs >= 1024 rows).  Graph of R calls over
disjoint cold regions (tools/cudatiming.py).  Usage: python tools/probes/rows_tiled_ab.py [row_bytes,row_bytes,...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls, disjoint_regions  # noqa: E402

dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)
TOTAL = 256 << 20
SIZES = [int(k) for k in sys.argv[1].split(',')] if len(sys.argv) > 1 else [1 << k for k in range(5, 19)]  # row bytes
for dtype, ops in (("float32", ("sum", "max", "sum_accurate")), ("int32", ("sum",)), ("float64", ("sum", "min"))):
    es = 8 if dtype == "float64" else 4
    pool = torch.empty((2 << 30) // es, dtype=getattr(torch, dtype), device=dev)
    pool.random_(-1000, 1000) if dtype == "int32" else pool.uniform_(-1, 1)
    rb.prepare(stream, pool.numel())
    for op in ops:
        for nbytes in SIZES:
            kb = nbytes / 1024
            cols = nbytes // es
            rows = TOTAL // nbytes
            old = 4 if nbytes <= 512 else (3 if nbytes <= 4096 else (1 if nbytes <= 16384 else 2))
            warm, timed = disjoint_regions(pool, 6, rows * cols, align_elems=256)
            outs = torch.empty(rows, dtype=pool.dtype, device=dev)
            row = {"dtype": dtype, "op": op, "row_kb": kb, "rows": rows}
            for name, g in (("old_group", old), ("tiled", 6), ("old_group2", old), ("tiled2", 6)):
                def launch(t, g=g):
                    rb.reduce_batched(t.view(rows, cols), op, out=outs, stream=stream, seg_group=g)
                us = time_calls(launch, warm, timed, stream, repeats=3) * 1e6
                row[name] = round(us, 2)
            best_old, best_new = min(row["old_group"], row["old_group2"]), min(row["tiled"], row["tiled2"])
            row["GBps_old"] = round(TOTAL / best_old / 1e3, 1)
            row["GBps_tiled"] = round(TOTAL / best_new / 1e3, 1)
            print(json.dumps(row), flush=True)
    del pool
    torch.cuda.empty_cache()
