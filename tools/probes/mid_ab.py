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
    "twopass_256x2": dict(grid_combine=2, block=256, unroll=2, grid=-1),
    "twopass_256x1": dict(grid_combine=2, block=256, unroll=1, grid=-1),
    "atomic_256x1": dict(grid_combine=1, block=256, unroll=1, grid=-1),
    "lastblock_256x2": dict(grid_combine=3, block=256, unroll=2, grid=-1),
    "cub": None,
}
try:
    from tests import cub as cubref
    cubref.lib()
except Exception:
    CANDS.pop("cub")
if "cub" in CANDS:  # size CUB's temp storage before any capture
    for k in range(18, 24):
        cubref.reduce(1, 0, pool.data_ptr(), 1 << k, out.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
sizes = (18, 19, 20, 21, 22, 23)
if os.environ.get("MID_AB_ONLY"):  # e.g. "auto,twopass_256x2,cub" and sizes "19,20"
    keep = os.environ["MID_AB_ONLY"].split(",")
    CANDS = {k: v for k, v in CANDS.items() if k in keep}
    sizes = tuple(int(v) for v in os.environ.get("MID_AB_SIZES", "19,20").split(","))
tag = sys.argv[1] if len(sys.argv) > 1 else ""
for k in sizes:
    m = 1 << k
    R = max(5, min(100, (400 << 20) // (4 * m)))
    warm, timed = disjoint_regions(pool, R, m)
    res = {c: [] for c in CANDS}
    for rnd in range(4):
        for name, kw in CANDS.items():
            ctr = [0]

            def launch(t, kw=kw):
                ctr[0] = (ctr[0] + 1) % 4096
                if kw is None:
                    cubref.reduce(1, 0, t.data_ptr(), t.numel(), out[ctr[0]:ctr[0] + 1].data_ptr(), s.cuda_stream)
                else:
                    rb.reduce(t, "sum", out=out[ctr[0]:ctr[0] + 1], stream=s, **kw)
            try:
                res[name].append(time_calls(launch, warm, timed, s, repeats=2) * 1e6)
            except Exception as e:
                res[name].append(float("nan"))
    print(json.dumps({"tag": tag, "log2_n": k, **{c: round(statistics.median(v), 3) for c, v in res.items()}}), flush=True)
