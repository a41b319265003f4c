"""A/B helper: batched aligned short rows (8 / 32 / 64 fp32 columns, 8 fp64
columns, 256 MB) per swapped library build.  Usage: python tools/probes/rows_ab.py TAG"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls  # noqa: E402

dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)
pool = torch.rand((256 << 20) // 4 + 64, device=dev)
row = {"tag": sys.argv[1] if len(sys.argv) > 1 else ""}
for dtype, cols in (("float32", 8), ("float32", 32), ("float32", 64), ("float64", 8), ("float64", 32)):
    tdt = getattr(torch, dtype)
    s = 8 if dtype == "float64" else 4
    rows = (256 << 20) // (s * cols)
    xv = pool.view(torch.uint8)[: rows * cols * s].view(tdt).view(rows, cols)
    ob = torch.empty(rows, dtype=tdt, device=dev)

    def launch(t, ob=ob, xv=xv):
        rb.reduce_batched(xv, "sum", out=ob, stream=stream)
    row[f"{dtype}x{cols}"] = round(time_calls(launch, [xv] * 3, [xv] * 10, stream, repeats=3) * 1e6, 2)
print(json.dumps(row), flush=True)
