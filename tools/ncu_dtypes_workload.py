"""The SURVEY 8(d) ncu evidence set: reduce() of 2^28 int32, 2^28 fp32 and
2^26 fp64 (sum, min, max; the bench's launch configuration from the dispatch
table), each twice (tools/profile_dtypes.sh skips the first launch of each)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402

dev = torch.device("cuda", 0)
buf = torch.rand((1 << 30) // 4, device=dev)
cases = [(buf.view(torch.int32), "int32"), (buf, "float32"), (buf.view(torch.float64)[: 1 << 26], "float64")]
for x, name in cases:
    for op in ("sum", "min", "max"):
        for _ in range(2):
            rb.reduce(x, op)
torch.cuda.synchronize()
print("dtype workload done")
