"""Host-side logic of the sharded mode (step S7) on CPU with the gloo backend,
world size 2 (the NCCL data path itself needs GPUs: tests/test_multi_gpu.py).

* the NCCL unique id made by rank 0 (reduce_comm_get_unique_id, CPU-only
  call) reaches every rank byte-identical through the torch process group;
* shard_range partitions [0, n) exactly, and combining the per-rank partial
  results in rank order (the deterministic-mode order; int32 as uint32 wrap,
  min/max by selection) reproduces the oracle of the whole array bit-exactly,
  for uneven and empty shards;
* invalid reduce_multi arguments are rejected before any NCCL/CUDA call.
"""
import ctypes
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_cgo_gonzalohghmh19_b200 as rb
        import oracle
        import synth
        uid = rb.broadcast_unique_id()
        uids = [None] * world
        dist.all_gather_object(uids, uid)
        res = {"uid_equal": all(u == uids[0] for u in uids), "uid_len": len(uid)}
        # partition + rank-order combine of per-rank partials == oracle(whole)
        checks = []
        for dtype in ("int32", "float32", "float64"):
            for n in (0, 1, 7, 1001, 65537):
                x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", 99 + n)
                lo, hi = rb.shard_range(n, world, rank)
                mine = x[lo:hi]
                parts = {}
                for op in ("sum", "min", "max"):
                    r = oracle.reduce(mine, op)
                    parts[op] = r.bits if r.bits is not None else r.value
                allp = [None] * world
                dist.all_gather_object(allp, (lo, hi, parts))
                cover = sorted((a, b) for a, b, _ in allp)
                ok_cover = cover[0][0] == 0 and cover[-1][1] == n and all(
                    cover[i][1] == cover[i + 1][0] for i in range(world - 1))
                for op in ("sum", "min", "max"):
                    whole = oracle.reduce(x, op)
                    vals = [p[op] for _, _, p in allp]
                    if dtype == "int32" and op == "sum":
                        comb = int(np.uint32(sum(int(np.uint32(np.int32(v).view(np.uint32))) for v in
                                                 [np.int32(np.uint32(b)) for b in vals]) % (1 << 32)))
                        checks.append((dtype, n, op, ok_cover and comb == whole.bits))
                    elif dtype == "int32":
                        iv = [int(np.uint32(b).view(np.int32)) for b in vals]
                        comb = int(np.int32(min(iv) if op == "min" else max(iv)).view(np.uint32))
                        checks.append((dtype, n, op, ok_cover and comb == whole.bits))
                    elif op != "sum":
                        w = 32 if dtype != "float64" else 64
                        fv = [np.array([b], dtype=np.uint32 if w == 32 else np.uint64).view(
                            np.float32 if w == 32 else np.float64)[0] for b in vals]
                        comb = oracle.reduce(np.array(fv, dtype=np.float32 if w == 32 else np.float64), op).bits
                        checks.append((dtype, n, op, ok_cover and comb == whole.bits))
                    else:
                        comb = sum(vals)
                        checks.append((dtype, n, op, ok_cover and abs(comb - whole.value) <= 1e-9 * (1 + whole.abs_sum)))
        res["checks"] = checks
        # argument validation without touching NCCL/CUDA
        st1 = rb.lib.reduce_multi(1, 0, None, 0, ctypes.c_void_p(4096), None, None)   # comm NULL
        st2 = rb.lib.reduce_multi(1, 0, None, 0, None, None, ctypes.c_void_p(8))      # out NULL
        st3 = rb.lib.reduce_multi(7, 0, None, 0, ctypes.c_void_p(4096), None, ctypes.c_void_p(8))
        res["invalid"] = (st1, st2, st3)
        q.put((rank, res))
        dist.destroy_process_group()
    except Exception as e:  # surface to the parent
        import traceback
        q.put((rank, {"error": traceback.format_exc()}))


def test_sharded_mode_host_logic_gloo_world2():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert "error" not in out[r], out[r].get("error")
        assert out[r]["uid_equal"] and out[r]["uid_len"] == 128
        bad = [c for c in out[r]["checks"] if not c[3]]
        assert not bad, bad
        assert out[r]["invalid"] == (1, 1, 1)
