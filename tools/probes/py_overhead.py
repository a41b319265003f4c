"""Host cost of one Python reduce() call (no sync): the binding's marshalling on
top of the C ABI.  Usage: python tools/probes/py_overhead.py TAG"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402

x = torch.rand(1024, device="cuda")
o = torch.empty(1, device="cuda")
s = torch.cuda.Stream()
res = {"tag": sys.argv[1] if len(sys.argv) > 1 else ""}
for name, kw in (("plain", {}), ("mode_kw", {"mode": "fast"})):
    for _ in range(1000):
        rb.reduce(x, "sum", out=o, stream=s, **kw)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(20000):
        rb.reduce(x, "sum", out=o, stream=s, **kw)
    res[name + "_us"] = round((time.perf_counter() - t0) / 20000 * 1e6, 3)
    torch.cuda.synchronize()
# the C ABI alone through ctypes (raw pointers, prebuilt arguments)
f = rb.lib.reduce
args = (1, 0, x.data_ptr(), x.numel(), o.data_ptr(), s.cuda_stream)
for _ in range(1000):
    f(*args)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(20000):
    f(*args)
res["ctypes_c_abi_us"] = round((time.perf_counter() - t0) / 20000 * 1e6, 3)
torch.cuda.synchronize()
print(json.dumps(res))
