"""Segmented (offsets-array) workloads for ncu: 256 MB of fp32 in segments of
power-law (mean 64), uniform 0..128 and uniform 0..2048 lengths, each through
reduce_segmented's auto path (element-balanced chunks) and run twice (the
profile skips the first, cold call).  Usage: python tools/segbal_workload.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402

dev = torch.device("cuda", 0)
x = torch.rand((256 << 20) // 4, device=dev)
rng = np.random.Generator(np.random.PCG64(7))
cases = []
for dist, mean in (("powerlaw", 64), ("uniform", 64), ("uniform", 1024)):
    nseg = x.numel() // mean
    if dist == "uniform":
        lens = rng.integers(0, 2 * mean + 1, nseg)
    else:
        lens = np.minimum((rng.pareto(1.2, nseg) * mean * 0.2).astype(np.int64) + 1, 1 << 20)
    offs = np.minimum(np.concatenate([[0], np.cumsum(lens)]), x.numel())
    cases.append((x[: int(offs[-1])], torch.from_numpy(offs).to(dev)))
for _ in range(2):
    for xv, ot in cases:
        rb.reduce_segmented(xv, ot, "sum")
torch.cuda.synchronize()
print("segbal workload done")
