"""Same-box A/B at large sizes (graph of calls on one resident array; > L2):
fp32 sum at 2^28 and 2^31 elements, fp64 min / max at 2^27.  Usage: TAG"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else ""
dev = torch.device("cuda", 0)
s = torch.cuda.Stream(dev)
x = torch.rand(1 << 31, dtype=torch.float32, device=dev, generator=torch.Generator(dev).manual_seed(2019))
rb.prepare(s, x.numel())
row = {"tag": tag}
for name, t, op in (("f32_sum_2^28", x[: 1 << 28], "sum"), ("f32_sum_2^31", x, "sum"),
                    ("f64_min_2^27", x[: 1 << 28].view(torch.float64), "min"),
                    ("f64_max_2^27", x[: 1 << 28].view(torch.float64), "max"),
                    ("i32_sum_2^28", x[: 1 << 28].view(torch.int32), "sum")):
    o = torch.empty(1, dtype=t.dtype, device=dev)
    reps = 5 if t.numel() > (1 << 29) else 20
    sec = time_calls(lambda r: rb.reduce(r, op, out=o, stream=s), [t] * 3, [t] * reps, s, repeats=3)
    row[name] = round(sec * 1e6, 2)
print(json.dumps(row), flush=True)
