"""One forced mid-size launch shape, repeated (for ncu source-level capture)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402

x = torch.rand(1 << 19, device="cuda")
o = torch.empty(1, device="cuda")
for _ in range(4):
    rb.reduce(x, "sum", out=o, grid_combine=2, block=256, unroll=2, grid=-1)
torch.cuda.synchronize()
