"""bench.py on the GPU: the N=1 line in the driver's contract shape, and the
multi-rank path (torchrun, 2 ranks) in --share-gpu test mode -- both ranks on
the one GPU, team combine over CUDA IPC, max-over-ranks timing -- so the code
the driver's 2/4/8-GPU scaling run executes is exercised here."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "roofline", "clocks", "gpu_launches")


def _one_line(r):
    assert r.returncode == 0, (r.stdout[-2000:], r.stderr[-3000:])
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_single_gpu_line():
    r = subprocess.run([sys.executable, "bench.py", "--steps", "5", "--warmup", "3", "--n", str(1 << 24),
                        "--no-sweep", "--no-cpu"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    d = _one_line(r)
    for k in KEYS + ("e2e",):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["gpu_launches"] >= 5
    assert d["roofline"]["bound"] == "hbm" and d["roofline"]["achieved"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == (1 << 24) * 4


def test_bench_two_ranks_share_gpu():
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr", "127.0.0.1", "--master-port", "29561", "bench.py", "--gpus", "2",
                        "--steps", "5", "--warmup", "3", "--elements", str(1 << 22), "--share-gpu"],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    d = _one_line(r)
    for k in KEYS:
        assert k in d, k
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["test_mode"]
    assert d["config"]["collective"] == "team" and d["config"]["parallelism"] == "shard2"
    assert "combine_us_per_step" in d["sharded_decomposition"]
    assert d["cross_rank_check"]["team"]["ok"], d["cross_rank_check"]
    assert d["comm"]["team_members"] == 2 and d["comm"]["world_size"] == 2


def test_bench_gpus_2_spawns_its_own_ranks():
    """`bench.py --gpus 2` outside torchrun re-executes itself under
    torch.distributed.run with 2 ranks (here both on the one GPU, --share-gpu)
    and reports both scaling series."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--steps", "4", "--warmup", "3",
                        "--elements", str(1 << 22), "--strong-total", str((1 << 23) + 5), "--share-gpu"],
                       capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    d = _one_line(r)
    assert d["n_gpus"] == 2 and d["scaling"] == "weak"
    st = d["strong_scaling"]
    assert st["total_elements"] == (1 << 23) + 5 and st["n_local_rank0"] == ((1 << 23) + 5) // 2
    assert st["value"] > 0 and st["cross_rank_check"]["ok"], st
    assert d["weak_scaling"]["n_per_gpu"] == 1 << 22
    assert d["cross_rank_check"]["team"]["ok"] and d["cross_rank_check"]["nccl"].startswith("unavailable")


def test_bench_strong_scaling_value():
    r = subprocess.run([sys.executable, "bench.py", "--steps", "4", "--warmup", "3", "--n", str(1 << 22),
                        "--strong-total", str(1 << 26), "--scaling", "strong", "--no-sweep", "--no-cpu", "--no-e2e"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    d = _one_line(r)
    assert d["scaling"] == "strong" and d["strong_scaling"]["total_elements"] == 1 << 26
    assert d["value"] == d["strong_scaling"]["value"] and d["config"]["total_bytes"] == 1 << 28
