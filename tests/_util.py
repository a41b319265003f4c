"""Shared helpers for the GPU parity tests: run the CUDA path through the C ABI
and compare with the oracle by DESIGN.md's rules (bit-exact for int32 and
min/max; gates G1 and G2 for fp sums)."""
from __future__ import annotations

import numpy as np

import oracle
from tests._chain import checked_chain

NP = {"int32": np.int32, "float32": np.float32, "float64": np.float64}
BITS = {"int32": np.uint32, "float32": np.uint32, "float64": np.uint64}


def to_device(x: np.ndarray, offset: int = 0):
    """Copy x to the GPU so that the returned tensor starts `offset` elements
    past a 256-byte-aligned allocation (exercises the misaligned head)."""
    import torch
    t = torch.empty(x.size + offset + 8, dtype=getattr(torch, x.dtype.name), device="cuda")
    v = t[offset:offset + x.size]
    if x.size:
        v.copy_(torch.from_numpy(np.ascontiguousarray(x)))
    return v


def gpu_reduce_many(cases, **opts):
    """cases: list of (device_tensor, op). Launch all, sync once, return the
    result bit patterns (numpy unsigned ints) and the plans."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    outs, plans = [], []
    for t, op in cases:
        out = torch.empty(1, dtype=t.dtype, device="cuda")
        rb.reduce(t, op, out=out, **opts)
        outs.append(out)
        plans.append(rb.query_plan(t.dtype.__str__().split(".")[-1], op, t.numel(), in_ptr=t.data_ptr(), **opts))
    torch.cuda.synchronize()
    res = [o.cpu().numpy() for o in outs]
    return res, plans


def check(x: np.ndarray, op: str, got: np.ndarray, plan: dict | None = None, gates=("g1", "g2")):
    """Assert the GPU result `got` (1-element array of x's dtype) matches the oracle."""
    dt = x.dtype.name
    ref = oracle.reduce(x, op)
    if dt == "int32" or op != "sum":
        gb = int(got.view(BITS[dt])[0])
        assert gb == ref.bits, f"{dt} {op} n={x.size}: got bits {gb:#x} want {ref.bits:#x} ({got[0]!r} vs {ref.value!r})"
        return
    # G2's L comes from the test-side formula over the plan's launch shape
    # (tests/_chain.py), never from the library's own plan["chain"]
    chain = checked_chain(dt, op, plan) if (plan is not None and "g2" in gates) else None
    ok, msg = oracle.check_sum(float(got[0]), ref, x.dtype, x.size, chain=chain)
    assert ok, f"{dt} sum n={x.size}: {msg} plan={plan}"
