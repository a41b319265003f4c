#!/usr/bin/env python
"""Device time per call (CUDA graph over cold regions, tools/cudatiming.py) of
CUB DeviceReduce vs this library (default dispatch + forced variants), fp32 sum.
Context for the paper's headline comparison (Tangram vs CUB)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))


def main():
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    from tests import cub
    from cudatiming import time_calls, disjoint_regions
    dev = torch.device("cuda", 0)
    s = torch.cuda.Stream(dev)
    pool = torch.rand((2 << 30) // 4, device=dev)
    rb.prepare(s, pool.numel())
    outs = torch.empty(4096, device=dev)
    variants = {"default": {}, "256x2 atomic": dict(block=256, unroll=2, grid_combine=1, grid=-1),
                "256x2 2pass": dict(block=256, unroll=2, grid_combine=2, grid=-1),
                "256x2 lastblk": dict(block=256, unroll=2, grid_combine=3, grid=-1),
                "256x4 atomic": dict(block=256, unroll=4, grid_combine=1, grid=-1),
                "cluster16 1024x2": dict(block=1024, unroll=2, grid_combine=4, grid=16)}
    rows = []
    for lb in range(16, 29, 2):
        n = 1 << lb
        R = max(5, min(100, (400 << 20) // (4 * n)))
        warm, timed = disjoint_regions(pool, R, n)
        ctr = [0]

        def lc(t):
            ctr[0] = (ctr[0] + 1) % 4096
            cub.reduce(1, 0, t.data_ptr(), n, outs[ctr[0]:ctr[0] + 1].data_ptr(), s.cuda_stream)
        cub.reduce(1, 0, timed[0].data_ptr(), n, outs.data_ptr(), s.cuda_stream)
        torch.cuda.synchronize()
        row = {"n": n, "cub_us": round(time_calls(lc, warm, timed, s, repeats=3) * 1e6, 3)}
        for name, kw in variants.items():
            opts = rb.make_opts(**kw) if kw else None

            def lo(t, opts=opts):
                ctr[0] = (ctr[0] + 1) % 4096
                rb.reduce_ptr(1, 0, t.data_ptr(), n, outs[ctr[0]:ctr[0] + 1].data_ptr(), s.cuda_stream, opts)
            try:
                row[name] = round(time_calls(lo, warm, timed, s, repeats=3) * 1e6, 3)
            except Exception as e:
                row[name] = str(e)[:40]
        rows.append(row)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
