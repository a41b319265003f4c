"""One call of each next-row workload at the bench's
sizes, for ncu (tools/profile_next_rows.sh): uniform batches of 64 / 1024 /
16384 fp32 columns (256 MB), power-law segments via offsets (256 MB) and the
256 / 65536-bin fp32 histograms of 2^28 elements.  Each workload runs twice;
the profile script skips the first (cold module / queue allocation)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402

dev = torch.device("cuda", 0)
x = torch.rand((256 << 20) // 4, device=dev)
rng = np.random.Generator(np.random.PCG64(7))
lens = np.minimum((rng.pareto(1.2, 1 << 20) * 12.8).astype(np.int64) + 1, 1 << 20)
offs = np.minimum(np.concatenate([[0], np.cumsum(lens)]), x.numel())
ot = torch.from_numpy(offs).to(dev)
xh = torch.rand(1 << 28, device=dev)
for _ in range(2):
    for cols in (64, 1024, 16384):
        rb.reduce_batched(x.view(-1, cols), "sum")
    rb.reduce_segmented(x[: int(offs[-1])], ot, "sum")
    for nb in (256, 65536):
        rb.histogram(xh, 0.0, 1.0, nb)
torch.cuda.synchronize()
print("next-rows workload done")
