"""Launch shapes and cold device times of CUB's DeviceReduce vs ours (run under
ncu).  Usage: python tools/probes/cub_shape.py [log2_n]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from tests import cub as cubref  # noqa: E402

k = int(sys.argv[1]) if len(sys.argv) > 1 else 20
x = torch.rand(1 << k, device="cuda")
o = torch.empty(1, device="cuda")
s = torch.cuda.current_stream()
for _ in range(3):
    cubref.reduce(1, 0, x.data_ptr(), x.numel(), o.data_ptr(), s.cuda_stream)
    rb.reduce(x, "sum", out=o, grid_combine=2, block=256, unroll=2, grid=-1)
    rb.reduce(x, "sum", out=o, grid_combine=1, block=256, unroll=4, grid=-1)
torch.cuda.synchronize()
print("done")
