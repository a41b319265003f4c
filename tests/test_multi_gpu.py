"""Sharded mode on real GPUs: reduce_multi over NCCL (world = number of visible
GPUs, capped at 8; the 1-GPU box runs world 1, which still exercises the
NCCL all-reduce / all-gather + finalise path end to end)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reduce_multi_matches_oracle_of_concatenation():
    import torch
    world = min(torch.cuda.device_count(), 8)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", "29517",
           os.path.join(ROOT, "tests", "multi_worker.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    assert r.returncode == 0 and len(lines) == world, (r.returncode, r.stdout[-2000:], r.stderr[-4000:])
    for l in lines:
        assert l["checked"] > 0 and not l["fails"], l
        assert l["deterministic_distinct"] == 1, l
