"""Pin P10: an independent implementation -- cub::DeviceReduce
from the CUDA 12.9 toolkit -- on the same device buffers.  int32 and fp min/max
bit-exact with ours (data without NaN / mixed signed zeros, where CUB's `<`
semantics are unspecified); fp sums: both within G2 of the oracle."""
import numpy as np
import pytest

import oracle
import synth
from tests._util import check, to_device

pytestmark = pytest.mark.gpu
DT = {"int32": 0, "float32": 1, "float64": 2}
OPC = {"sum": 0, "min": 1, "max": 2}


@pytest.mark.parametrize("dtype", ["int32", "float32", "float64"])
def test_cub_agrees(dtype):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    from tests import cub
    for k, n in enumerate([1, 1000, 65537, (1 << 22) + 3, 1 << 26]):
        x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", 600 + k)
        t = to_device(x, k % 4)
        for op in ("sum", "min", "max"):
            mine = rb.reduce(t, op)
            theirs = torch.empty_like(mine)
            cub.reduce(DT[dtype], OPC[op], t.data_ptr(), n, theirs.data_ptr(),
                       torch.cuda.current_stream().cuda_stream)
            torch.cuda.synchronize()
            a, b = mine.cpu().numpy(), theirs.cpu().numpy()
            if dtype == "int32" or op != "sum":
                assert a.tobytes() == b.tobytes(), (dtype, op, n, a, b)
            else:
                plan = rb.query_plan(dtype, op, n, in_ptr=t.data_ptr())
                check(x, op, a, plan)
                ok, msg = oracle.check_sum(float(b[0]), oracle.reduce(x, "sum"), x.dtype, n)
                assert ok, ("cub", msg)
