"""Per-kernel device time of the element-balanced segmented path in a graph
(the three kernels separately): REDUCE_SEGBAL_ONLY = all | scan | main | fix
selects which of the three each call launches (read per call by the library once
set); each partial call reuses what the full call before it left in the
workspace.  Usage: python tools/probes/segbal_split.py"""
import json
import os
os.environ["REDUCE_SEGBAL_ONLY"] = "all"  # before the library's first segmented call
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls  # noqa: E402

dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)
rb.prepare(stream, 1 << 20)
total = 256 << 20
pool = torch.rand(total // 4 + 64, device=dev)
rng = np.random.Generator(np.random.PCG64(7))
for dist, mean in (("uniform", 64), ("uniform", 1024), ("powerlaw", 64)):
    nseg = total // 4 // mean
    lens = rng.integers(0, 2 * mean + 1, nseg) if dist == "uniform" else \
        np.minimum((rng.pareto(1.2, nseg) * mean * 0.2).astype(np.int64) + 1, 1 << 20)
    offs = np.minimum(np.concatenate([[0], np.cumsum(lens)]), total // 4)
    ot = torch.from_numpy(offs).to(dev)
    x = pool[: int(offs[-1])]
    ob = torch.empty(nseg, dtype=torch.float32, device=dev)

    def launch(t, ob=ob, x=x, ot=ot):
        rb.reduce_segmented(x, ot, "sum", out=ob, stream=stream)
    for only in ("all", "scan", "main", "fix", "all"):
        os.environ["REDUCE_SEGBAL_ONLY"] = "all"
        launch(x)  # a full call: the workspace holds this input's chunk arrays
        os.environ["REDUCE_SEGBAL_ONLY"] = only
        sec = time_calls(launch, [x] * 3, [x] * 10, stream, repeats=3)
        print(json.dumps({"dist": dist, "mean_len": mean, "only": only, "us": round(sec * 1e6, 2)}))
    os.environ["REDUCE_SEGBAL_ONLY"] = "all"
