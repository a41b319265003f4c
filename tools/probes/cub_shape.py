"""Launch shapes of CUB's DeviceReduce vs ours at 1 M fp32 (run under ncu)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from tests import cub as cubref  # noqa: E402

x = torch.rand(1 << 20, device="cuda")
o = torch.empty(1, device="cuda")
s = torch.cuda.current_stream()
for _ in range(3):
    cubref.reduce(1, 0, x.data_ptr(), x.numel(), o.data_ptr(), s.cuda_stream)
    rb.reduce(x, "sum", out=o)
torch.cuda.synchronize()
print("done")
