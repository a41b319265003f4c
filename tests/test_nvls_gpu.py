"""The NVLS (NVLink SHARP multicast) cross-GPU combine of reduce_multi_nvls on
the one-GPU box: a one-member multicast team made with the CUDA driver's
multicast API (reduce_nvls_create_local) runs the very kernels and protocol
of the k-GPU case -- mode 1: slot store, multimem.red barrier, multimem.ld_reduce
through the multicast object; mode 2: multimem.st of {word, epoch} pairs and
the rank-order combine -- so every dtype / op / grid combine is checked against
the oracle, over many back-to-back calls (epochs, parities and the barrier
counter advance) and graph replays.  The NCCL-built team (reduce_nvls_create)
is covered by tests/test_multi_gpu.py."""
import numpy as np
import pytest

import oracle
import synth
from tests._util import to_device

pytestmark = pytest.mark.gpu
OPS = ("sum", "min", "max")


def _rb():
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    return rb


@pytest.fixture(params=[1, 2], ids=["ld_reduce", "mcast_store"])
def nvls(request):
    rb = _rb()
    try:
        nv = rb.Nvls.local(mode=request.param)
    except rb.ReduceError as e:
        if e.status == 2:
            pytest.skip(f"no multicast on this device: {e}")
        raise
    yield nv
    import torch
    torch.cuda.synchronize()
    nv.destroy()


def _check(x, op, got):
    ref = oracle.reduce(x, "sum" if op == "sum_accurate" else op)
    dt = x.dtype.name
    if dt == "int32" or op not in ("sum", "sum_accurate"):
        bits = int(got.view(np.uint32 if dt != "float64" else np.uint64)[0])
        assert bits == ref.bits, (dt, op, x.size, bits, ref.bits)
    else:
        ok, msg = oracle.check_sum(float(got[0]), ref, x.dtype, max(x.size, 1))
        assert ok, (dt, op, x.size, msg)


@pytest.mark.parametrize("dtype", ["int32", "float32", "float64"])
def test_nvls_local_team_matches_oracle(nvls, dtype):
    rb = _rb()
    ops = OPS + (("sum_accurate",) if dtype != "int32" else ())
    variants = (dict(), dict(mode="deterministic"), dict(grid_combine=0, block=256), dict(grid_combine=1),
                dict(grid_combine=2), dict(grid_combine=3), dict(grid_combine=4, grid=16))
    for n in (0, 1, 1000, (1 << 20) + 7):
        x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", 300 + n)
        t = to_device(x, 1)
        for op in ops:
            for v in variants:
                if op == "sum_accurate" and dtype == "float64" and v.get("grid_combine") == 1:
                    continue
                got = rb.reduce_multi_nvls(t, op, nvls, **v).cpu().numpy()
                _check(x, op, got)


def test_nvls_local_team_back_to_back_and_graph(nvls):
    """Hundreds of calls in a row on one stream (the epoch, the parity slots and
    the barrier counter advance every call), then a captured graph replayed
    with fresh inputs."""
    import torch
    rb = _rb()
    s = torch.cuda.Stream()
    rb.prepare(s, 1 << 20)
    xs = [torch.full((1 << 16,), k + 1, dtype=torch.int32, device="cuda") for k in range(8)]
    res = torch.empty(800, dtype=torch.int32, device="cuda")
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        for i in range(800):
            rb.reduce_multi_nvls(xs[i % 8], "sum", nvls, out=res[i:i + 1], stream=s)
    torch.cuda.synchronize()
    assert (res.cpu().numpy() == np.array([(i % 8 + 1) << 16 for i in range(800)])).all()
    # graph: 4 calls captured, replayed 6 times with new inputs
    xin = torch.empty(1 << 16, dtype=torch.float32, device="cuda")
    gout = torch.empty(4, dtype=torch.float32, device="cuda")
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for j in range(4):
            rb.reduce_multi_nvls(xin, "max", nvls, out=gout[j:j + 1], stream=s)
    for rep in range(6):
        xin.copy_(torch.arange(1 << 16, dtype=torch.float32, device="cuda") * (rep + 1))
        with torch.cuda.stream(s):
            g.replay()
        torch.cuda.synchronize()
        assert (gout.cpu().numpy() == float(((1 << 16) - 1) * (rep + 1))).all(), rep
