"""Throwaway (not product code): launch one forced variant a few times (for ncu).
  python tools/probes/probe_one.py float64 max '{"grid":-1,"block":256,"unroll":4,"grid_combine":1}'"""
import json, sys, torch
import paper_conf_cgo_gonzalohghmh19_b200 as rb
dt, op, kw = sys.argv[1], sys.argv[2], json.loads(sys.argv[3])
x = torch.randn((1 << 30) // 8, dtype=torch.float64, device="cuda").view(getattr(torch, dt))
for _ in range(4):
    rb.reduce(x, op, **kw)
torch.cuda.synchronize()
