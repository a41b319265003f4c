"""Probe: launch configs and per-kernel device time of CUB vs ours at a few sizes (run under ncu)."""
import sys
sys.path.insert(0, ".")
import torch
import paper_conf_cgo_gonzalohghmh19_b200 as rb
from tests import cub
for n in (1 << 20, 1 << 22, 1 << 24):
    x = torch.rand(n, device="cuda")
    o = torch.empty(1, device="cuda")
    for _ in range(3):
        cub.reduce(1, 0, x.data_ptr(), n, o.data_ptr(), torch.cuda.current_stream().cuda_stream)
        rb.reduce(x, "sum", out=o)
        rb.reduce(x, "sum", out=o, mode="deterministic")
    torch.cuda.synchronize()
