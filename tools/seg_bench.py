"""Device time of the segmented / batched reductions on B200.

Prints one JSON line per case: uniform batches of short to long rows (the
bench's 256 MB batches) in each dtype, and variable-length segments (uniform
and power-law lengths) through reduce_segmented.  Graph-timed with CUDA events
(tools/cudatiming.py); every batch is larger than L2, so each call reads HBM.
Usage: python tools/seg_bench.py [--tag TAG]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))


GROUPS = {0: "auto", 1: "warp", 2: "block", 3: "8-lane", 4: "thread"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="")
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", default="", help="batched | segmented | histogram (default: all)")
    args = ap.parse_args()
    import numpy as np
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    from cudatiming import time_calls

    dev = torch.device("cuda", 0)
    stream = torch.cuda.Stream(dev)
    rb.prepare(stream, 1 << 20)  # workspace + segment queue before the graph captures
    total_bytes = 256 << 20
    pool = torch.rand(total_bytes // 4 + 64, device=dev)
    cases = []
    cols_list = (8, 32, 64, 100, 256, 1024, 16384) if not args.quick else (64, 1024)
    for dtype, op in (("float32", "sum"), ("int32", "sum"), ("float64", "sum"), ("float32", "max"),
                      ("float32", "sum_accurate")):
        if args.only and args.only != "batched":
            break
        if args.quick and dtype != "float32":
            continue
        tdt = getattr(torch, dtype)
        s = torch.empty(0, dtype=tdt).element_size()
        for cols in cols_list:
            rows = total_bytes // (s * cols)
            xv = pool.view(torch.uint8)[: rows * cols * s].view(tdt).view(rows, cols)
            ob = torch.empty(rows, dtype=tdt, device=dev)
            for group in (0, 1, 3, 4):
                def launch(t, ob=ob, xv=xv, group=group, op=op):
                    rb.reduce_batched(xv, op, out=ob, stream=stream, seg_group=group)
                sec = time_calls(launch, [xv] * 3, [xv] * 10, stream, repeats=2)
                cases.append({"kind": "batched", "dtype": dtype, "op": op, "rows": rows, "cols": cols,
                              "group": GROUPS[group], "us": round(sec * 1e6, 2),
                              "GBps": round(rows * cols * s / sec / 1e9, 1)})
    rng = np.random.Generator(np.random.PCG64(7))
    for dist, mean in (("uniform", 64), ("uniform", 1024), ("powerlaw", 64)):
        if args.only and args.only != "segmented":
            break
        nseg = total_bytes // 4 // mean
        if dist == "uniform":
            lens = rng.integers(0, 2 * mean + 1, nseg)
        else:
            lens = np.minimum((rng.pareto(1.2, nseg) * mean * 0.2).astype(np.int64) + 1, 1 << 20)
        offs = np.zeros(nseg + 1, np.int64)
        offs[1:] = np.cumsum(lens)
        offs = np.minimum(offs, total_bytes // 4)
        ot = torch.from_numpy(offs).to(dev)
        x = pool[: int(offs[-1])]
        ob = torch.empty(nseg, dtype=torch.float32, device=dev)
        for group in (0, 1, 2, 3, 4):
            def launch(t, ob=ob, x=x, ot=ot, group=group):
                rb.reduce_segmented(x, ot, "sum", out=ob, stream=stream, seg_group=group)
            sec = time_calls(launch, [x] * 3, [x] * 10, stream, repeats=2)
            cases.append({"kind": "segmented", "dist": dist, "mean_len": mean, "nseg": nseg,
                          "group": GROUPS[group], "us": round(sec * 1e6, 2),
                          "GBps": round(int(offs[-1]) * 4 / sec / 1e9, 1)})
    # histogram (N4): 1 GiB-class fp32 / int32 inputs, a range of bin counts
    xh = torch.rand(1 << 28, device=dev)
    xi = (xh * 2000 - 1000).to(torch.int32)
    for dtype, t, lo, hi in (("float32", xh, 0.0, 1.0), ("int32", xi, -1000.0, 1001.0)):
        if args.only and args.only != "histogram":
            break
        for nbins in (1, 4, 16, 64, 256, 512, 1024, 4096, 16384, 65536):
            if args.quick and nbins not in (256, 65536):
                continue
            hc = torch.empty(nbins, dtype=torch.int32, device=dev)

            def launch_h(tt, hc=hc, nbins=nbins, t=t, lo=lo, hi=hi):
                rb.histogram(t, lo, hi, nbins, counts=hc, stream=stream)
            sec = time_calls(launch_h, [t] * 2, [t] * 5, stream, repeats=2)
            cases.append({"kind": "histogram", "dtype": dtype, "n": t.numel(), "nbins": nbins,
                          "us": round(sec * 1e6, 2), "GBps": round(t.numel() * 4 / sec / 1e9, 1)})
    for c in cases:
        c["tag"] = args.tag
        print(json.dumps(c), flush=True)


if __name__ == "__main__":
    main()
