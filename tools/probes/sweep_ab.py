"""Per-call device time of the auto-dispatched reduce over a size sweep (graph
of R calls over disjoint cold regions, tools/tune.py's harness): for A/B of
library builds swapped in by tools/probes/lib_ab.sh.
Usage: python tools/probes/sweep_ab.py TAG [--input-ready]
(--input-ready: every call passes REDUCE_FLAG_INPUT_READY -- the inputs are
written once, long before -- so early register loads are allowed)"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls, disjoint_regions  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else ""
kw = dict(input_ready=True) if "--input-ready" in sys.argv else {}
dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)
for dtype, ops in (("float32", ("sum",)), ("int32", ("sum", "max")), ("float64", ("max",))):
    es = 8 if dtype == "float64" else 4
    pool = torch.empty((2 << 30) // es, dtype=getattr(torch, dtype), device=dev)
    pool.random_(-1000, 1000) if dtype == "int32" else pool.uniform_(-1, 1)
    rb.prepare(stream, pool.numel())
    out = torch.empty(4096, dtype=pool.dtype, device=dev)
    for op in ops:
        row = {"tag": tag, "dtype": dtype, "op": op}
        for lb in range(14, 31, 2):
            n = (1 << lb) // es
            R = max(20, min(100, (400 << 20) // (1 << lb))) if (1 << lb) >= (256 << 20) else max(5, min(100, (400 << 20) // (1 << lb)))
            warm, timed = disjoint_regions(pool, R, n)
            k = [0]

            def launch(t):
                i = k[0] = (k[0] + 1) % 4096
                rb.reduce(t, op, out=out[i:i + 1], stream=stream, **kw)
            row[f"2^{lb}"] = round(time_calls(launch, warm, timed, stream, repeats=3) * 1e6, 3)
        print(json.dumps(row), flush=True)
    del pool
    torch.cuda.empty_cache()
