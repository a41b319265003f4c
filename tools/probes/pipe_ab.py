"""1 GiB fp32 sum, graph-timed, at forced launch shapes (persistent grids and the
default): A/B of the rolling tile loop (RB_PIPE_TILES).  Usage: python
tools/probes/pipe_ab.py TAG"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else ""
dev = torch.device("cuda", 0)
s = torch.cuda.Stream(dev)
rb.prepare(s, 1 << 28)
x = torch.rand(1 << 28, device=dev)
out = torch.empty(1, device=dev)
shapes = [dict()] + [dict(grid=g, block=b, unroll=u, grid_combine=1)
                     for (g, b, u) in ((148 * 4, 256, 4), (148 * 5, 256, 4), (148 * 8, 256, 4), (148 * 2, 512, 4),
                                       (148 * 16, 256, 4), (148 * 2, 256, 8), (148 * 4, 256, 8), (148 * 1, 512, 8))]
for sh in shapes:
    def launch(t, sh=sh):
        rb.reduce(x, "sum", out=out, stream=s, **sh)
    sec = time_calls(launch, [x] * 3, [x] * 20, s, repeats=3)
    print(json.dumps({"shape": sh or "auto", "us": round(sec * 1e6, 2), "GBps": round(x.numel() * 4 / sec / 1e9, 1),
                      "tag": tag}))
