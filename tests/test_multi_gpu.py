"""Sharded mode on real GPUs: reduce_multi over NCCL (world = number of visible
GPUs, capped at 8; the 1-GPU box runs world 1, which still exercises the
NCCL all-reduce / all-gather + finalise path end to end), and the NVLS
combine (reduce_multi_nvls): parity where multicast exists, a clean
REDUCE_ERR_UNSUPPORTED where it does not."""
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
        assert l["comm_after_nvls"] == 1000.0 * world, l
        for mode, r in l["nvls"].items():
            if r["status"] == 0:   # NVLS multicast available: parity like reduce_multi
                assert r["checked"] > 0 and not r["fails"], (mode, r)
            else:                  # e.g. the 1-GPU box: a clean REDUCE_ERR_UNSUPPORTED
                assert r["status"] == 2, (mode, r)
    # every rank took the same branch
    assert len({json.dumps({m: r["status"] for m, r in l["nvls"].items()}) for l in lines}) == 1
