import sys; sys.path.insert(0, ".")
import torch, numpy as np
import paper_conf_cgo_gonzalohghmh19_b200 as rb
VARIANTS = [dict(), dict(mode="deterministic"), dict(grid_combine=0, block=256), dict(grid_combine=2),
            dict(grid_combine=3), dict(grid_combine=4, grid=16), dict(stage="smem", unroll=8, block=256),
            dict(block_combine=3, block=128), dict(grid=148, grid_combine=3)]
for n in [1, 7, 1000, 4097, (1 << 18) + 5, (1 << 21) + 3]:
    t = torch.ones(n, dtype=torch.float64, device="cuda")
    for v in VARIANTS:
        try:
            rb.reduce(t, "sum_accurate", **v).item()
        except Exception as e:
            print(n, v, rb.query_plan("float64", "sum_accurate", n, in_ptr=t.data_ptr(), **v), str(e)[:100])
