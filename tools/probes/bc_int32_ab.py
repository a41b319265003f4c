"""int32 block combines at the dispatch table's own launch shapes: the table
uses Vs (shuffle/redux + shared partials) everywhere; the variant study at a
fixed 256 x 2 shape ranked VA1 (per-thread shared atomic, warp-aggregated by
the compiler for integers) first.  This times, per size, the table's config
with block_combine = Vs / VA2+S / VA1 (graph-timed, cold regions, tools/tune.py's
harness).  Usage: python tools/probes/bc_int32_ab.py [int32|float32] [ops,comma-separated]"""
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
DTYPE = sys.argv[1] if len(sys.argv) > 1 else "int32"
OPS = sys.argv[2].split(",") if len(sys.argv) > 2 else ["sum", "max"]
DTC = {"int32": 0, "float32": 1, "float64": 2}[DTYPE]
pool = torch.empty((2 << 30) // (8 if DTYPE == "float64" else 4), dtype=getattr(torch, DTYPE), device=dev)
if DTYPE == "int32":
    pool.random_(-1000, 1000)
else:
    pool.uniform_(-1, 1)
rb.prepare(stream, pool.numel())
out = torch.empty(4096, dtype=pool.dtype, device=dev)
for op in OPS:
    for lb in range(12, 31, 2):
        n = (1 << lb) // (8 if DTYPE == "float64" else 4)
        R = max(20, min(100, (400 << 20) // (1 << lb))) if (1 << lb) >= (256 << 20) else max(5, min(100, (400 << 20) // (1 << lb)))
        warm, timed = disjoint_regions(pool, R, n)
        plan = rb.query_plan(DTYPE, op, n, in_ptr=pool.data_ptr())
        if plan["grid_combine"] == 4 or plan["grid_combine"] == 0:
            base = dict(block=plan["block"], unroll=plan["unroll"], grid_combine=plan["grid_combine"],
                        grid=plan["grid"] if plan["grid_combine"] == 4 else -1, stage=plan["stage"])
        else:
            base = dict(block=plan["block"], unroll=plan["unroll"], grid_combine=plan["grid_combine"], grid=-1,
                        stage=plan["stage"])
        row = {"dtype": DTYPE, "op": op, "bytes": f"2^{lb}", "plan": base}
        for bc, name in ((0, "Vs"), (1, "VA2+S"), (2, "VA1"), (3, "V")):
            opts = rb.make_opts(mode="fast", block_combine=bc, **base)
            k = [0]

            def launch(t, opts=opts):
                i = k[0] = (k[0] + 1) % 4096
                rb.reduce_ptr(DTC, op, t.data_ptr(), t.numel(), out[i:i + 1].data_ptr(), stream.cuda_stream, opts)
            try:
                row[name] = round(time_calls(launch, warm, timed, stream, repeats=3) * 1e6, 3)
            except Exception as e:
                row[name] = str(e)[:60]
        print(json.dumps(row), flush=True)
