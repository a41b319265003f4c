"""Same-box A/B of the grid combines at 8-128 MB (fp32 sum, graph of calls over
cold regions): ATOMIC vs FLAGS at a few launch shapes.  Usage: TAG"""
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
dev = torch.device("cuda", 0)
s = torch.cuda.Stream(dev)
pool = torch.rand(1 << 29, dtype=torch.float32, device=dev)
rb.prepare(s, pool.numel())
o = torch.empty(4096, dtype=torch.float32, device=dev)
shapes = [("A256x4", dict(grid_combine=1, block=256, unroll=4)), ("F256x4", dict(grid_combine=5, block=256, unroll=4)),
          ("F512x8", dict(grid_combine=5, block=512, unroll=8)), ("A512x4p296", dict(grid_combine=1, block=512, unroll=4, grid=296)),
          ("F512x4p296", dict(grid_combine=5, block=512, unroll=4, grid=296)),
          ("F256x4p1184", dict(grid_combine=5, block=256, unroll=4, grid=1184))]
for lb in (23, 24, 25, 26, 27):
    n = (1 << lb) // 4
    R = max(10, min(100, (400 << 20) // (1 << lb)))
    warm, timed = disjoint_regions(pool, R, n)
    row = {"tag": tag, "lb": lb}
    for name, kw in shapes:
        opts = rb.make_opts(**kw)
        k = [0]

        def launch(t, opts=opts):
            i = k[0] = (k[0] + 1) % 4096
            rb.reduce_ptr(1, "sum", t.data_ptr(), t.numel(), o[i:i + 1].data_ptr(), s.cuda_stream, opts)
        best = min(time_calls(launch, warm, timed, s, repeats=1) for _ in range(3))
        row[name] = round(best * 1e6, 2)
    print(json.dumps(row), flush=True)
