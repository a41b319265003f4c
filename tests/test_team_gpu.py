"""Sharded mode with the cross-GPU combine fused into the kernel (SURVEY 8(f)
N2, reduce_multi_team).  On the one-GPU box the team members are (a) streams of
one process (plain pointers) and (b) two processes sharing the GPU through CUDA
IPC handles -- the same peer-store / flag protocol that runs over NVLink between
GPUs.  Every member's result must equal the oracle of the concatenated shards
(bit-exact for int32 and min/max, G1 for sums) and be bit-identical across
members; repeated calls exercise the epoch / parity double buffering."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NP = {"int32": np.int32, "float32": np.float32, "float64": np.float64}
BITS = {"int32": np.uint32, "float32": np.uint32, "float64": np.uint64}


def _check_all(x, op, outs):
    dt = x.dtype.name
    ref = oracle.reduce(x, "sum" if op == "sum_accurate" else op)
    bits = {int(o.view(BITS[dt])[0]) for o in outs}
    assert len(bits) == 1, ("members disagree", dt, op, bits)
    if dt == "int32" or op not in ("sum", "sum_accurate"):
        assert bits.pop() == ref.bits, (dt, op)
    else:
        ok, msg = oracle.check_sum(float(outs[0][0]), ref, x.dtype, max(x.size, 1))
        assert ok, (dt, op, msg)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_team_streams_in_process(k):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    team = rb.Team.local(k)
    streams = [torch.cuda.Stream() for _ in range(k)]
    try:
        call = 0
        for dtype in ("int32", "float32", "float64"):
            for n in (0, 5, 1000, (1 << 20) + 3, (1 << 23) + 17):
                x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", 31 * n + k)
                shards = []
                for r in range(k):
                    lo, hi = rb.shard_range(n, k, r)
                    t = torch.empty(hi - lo + 1, dtype=getattr(torch, dtype), device="cuda")[1:]
                    if hi > lo:
                        t.copy_(torch.from_numpy(x[lo:hi]))
                    shards.append(t)
                torch.cuda.synchronize()
                ops = ("sum", "min", "max") + (("sum_accurate",) if dtype != "int32" else ())
                for op in ops:
                    for kw in (dict(), dict(mode="deterministic"), dict(grid_combine=3), dict(grid_combine=4, grid=8)):
                        outs = []
                        for r in range(k):
                            with torch.cuda.stream(streams[r]):
                                outs.append(rb.reduce_multi_team(shards[r], op, team[r], stream=streams[r], **kw))
                        call += 1
                        torch.cuda.synchronize()
                        _check_all(x, op, [o.cpu().numpy() for o in outs])
        assert call > 50
    finally:
        torch.cuda.synchronize()
        for t in team:
            t.destroy()


def test_team_same_gpu_back_to_back():
    """Two members on one GPU, 40 calls each queued on their streams with no
    host sync in between (large grids, so programmatic dependent launch would
    let the next call's CTAs park on the SMs): members sharing a GPU do not
    trigger early, so neither member can starve the other out of the exchange."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    k, n, iters = 2, (1 << 25) + 3, 40
    team = rb.Team.local(k)
    streams = [torch.cuda.Stream() for _ in range(k)]
    try:
        x = synth.make("float32", n, "uniform_pm1", 4242)
        shards = []
        for r in range(k):
            lo, hi = rb.shard_range(n, k, r)
            shards.append(torch.from_numpy(x[lo:hi]).cuda())
        outs = [[torch.empty(1, device="cuda") for _ in range(iters)] for _ in range(k)]
        torch.cuda.synchronize()
        for it in range(iters):
            for r in range(k):
                rb.reduce_multi_team(shards[r], "sum", team[r], out=outs[r][it], stream=streams[r])
        torch.cuda.synchronize()
        for it in range(iters):
            _check_all(x, "sum", [outs[r][it].cpu().numpy() for r in range(k)])
    finally:
        torch.cuda.synchronize()
        for t in team:
            t.destroy()


def test_team_graph_replay():
    """Team calls captured once per member into CUDA graphs and replayed: the
    epoch is advanced on the device, so every replay is a fresh exchange (new
    input values must show up in every member's result)."""
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    k, n = 2, (1 << 20) + 11
    team = rb.Team.local(k)
    streams = [torch.cuda.Stream() for _ in range(k)]
    try:
        shards, outs, graphs = [], [], []
        for r in range(k):
            lo, hi = rb.shard_range(n, k, r)
            shards.append(torch.zeros(hi - lo, dtype=torch.int32, device="cuda"))
            outs.append(torch.zeros(1, dtype=torch.int32, device="cuda"))
        torch.cuda.synchronize()
        for r in range(k):  # warm (first call allocates the stream's workspace)
            rb.reduce_multi_team(shards[r], "sum", team[r], out=outs[r], stream=streams[r])
        torch.cuda.synchronize()
        for r in range(k):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=streams[r]):
                rb.reduce_multi_team(shards[r], "sum", team[r], out=outs[r], stream=streams[r])
            graphs.append(g)
        torch.cuda.synchronize()
        for rep in range(6):
            x = synth.make("int32", n, "int_full", 500 + rep)
            for r in range(k):
                lo, hi = rb.shard_range(n, k, r)
                shards[r].copy_(torch.from_numpy(x[lo:hi]))
            torch.cuda.synchronize()
            for r in range(k):
                with torch.cuda.stream(streams[r]):
                    graphs[r].replay()
            torch.cuda.synchronize()
            _check_all(x, "sum", [o.cpu().numpy() for o in outs])
    finally:
        torch.cuda.synchronize()
        for t in team:
            t.destroy()


def test_team_two_processes_ipc():
    script = os.path.join(ROOT, "tests", "team_ipc_worker.py")
    world = 2
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
                        "--master-addr", "127.0.0.1", "--master-port", "29551", script],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    lines, dec = [], json.JSONDecoder()
    for l in r.stdout.splitlines():
        while l.startswith("{"):
            obj, end = dec.raw_decode(l)
            lines.append(obj)
            l = l[end:].lstrip()
    assert r.returncode == 0 and len(lines) == world, (r.returncode, r.stdout[-2000:], r.stderr[-3000:])
    for l in lines:
        assert l["checked"] > 0 and not l["fails"], l
