"""Throwaway A/B probe (not product code): device time per call of forced
variants of one (dtype, op) at 1 GiB, cold inputs, CUDA-graph timed.  Run with
PYTHONPATH pointing at a copy of the package built with a variant.
  python tools/probes/probe_ab_ops.py float64 max"""
import sys, os
import torch
import paper_conf_cgo_gonzalohghmh19_b200 as rb
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
from cudatiming import time_calls, disjoint_regions

dt, op = sys.argv[1], sys.argv[2]
tdt = getattr(torch, dt)
es = torch.empty(0, dtype=tdt).element_size()
pool = torch.randn((6 << 30) // 8, dtype=torch.float64, device="cuda").view(tdt)
n = (1 << 30) // es
w, t = disjoint_regions(pool, 2, n)
out = torch.empty(16, dtype=tdt, device="cuda")
s = torch.cuda.Stream()
rb.prepare(s, n)
shapes = [dict(), dict(grid=296, block=256, unroll=4), dict(grid=592, block=256, unroll=4),
          dict(grid=-1, block=256, unroll=4), dict(grid=-1, block=512, unroll=4), dict(grid=-1, block=256, unroll=2),
          dict(grid=-1, block=1024, unroll=2), dict(grid=-1, block=128, unroll=8)]
if len(sys.argv) > 3:
    import json
    shapes = json.loads(sys.argv[3])
print(rb.__file__)
for kw in shapes:
    try:
        sec = time_calls(lambda x, kw=kw: rb.reduce(x, op, out=out[:1], stream=s, **kw), w, t, s, repeats=3)
        print(f"{dt} {op} {str(kw):45s} {n*es/sec/1e9:8.1f} GB/s")
    except Exception as e:
        print(f"{dt} {op} {str(kw):45s} error {e}")
