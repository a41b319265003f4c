"""Same-box A/B of launch shapes at medium sizes (graph of calls over cold
regions), alternating the candidates several rounds.  Usage: python tools/probes/mid_ab.py"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls, disjoint_regions  # noqa: E402

dev = torch.device("cuda", 0)
s = torch.cuda.Stream(dev)
pool = torch.rand((1 << 30) // 4, device=dev)
rb.prepare(s, pool.numel())
out = torch.empty(4096, device=dev)
CANDS = {
    "auto": {},
    "atomic_128x4": dict(grid_combine=1, block=128, unroll=4, grid=-1),
    "atomic_256x4": dict(grid_combine=1, block=256, unroll=4, grid=-1),
    "atomic_512x4": dict(grid_combine=1, block=512, unroll=4, grid=-1),
    "atomic_256x2": dict(grid_combine=1, block=256, unroll=2, grid=-1),
    "twopass_128x4": dict(grid_combine=2, block=128, unroll=4, grid=-1),
    "twopass_128x8": dict(grid_combine=2, block=128, unroll=8, grid=-1),
    "lastblock_256x4": dict(grid_combine=3, block=256, unroll=4, grid=-1),
    "cluster16_1024x4": dict(grid_combine=4, block=1024, unroll=4, grid=16),
}
for k in (18, 19, 20, 21, 22, 23):
    m = 1 << k
    R = max(5, min(100, (400 << 20) // (4 * m)))
    warm, timed = disjoint_regions(pool, R, m)
    res = {c: [] for c in CANDS}
    for rnd in range(4):
        for name, kw in CANDS.items():
            ctr = [0]

            def launch(t, kw=kw):
                ctr[0] = (ctr[0] + 1) % 4096
                rb.reduce(t, "sum", out=out[ctr[0]:ctr[0] + 1], stream=s, **kw)
            try:
                res[name].append(time_calls(launch, warm, timed, s, repeats=2) * 1e6)
            except Exception as e:
                res[name].append(float("nan"))
    print(json.dumps({"log2_n": k, **{c: round(statistics.median(v), 3) for c, v in res.items()}}), flush=True)
