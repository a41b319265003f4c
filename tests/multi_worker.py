"""Worker for tests/test_multi_gpu.py (run under torch.distributed.run, one rank
per GPU, NCCL).  Every rank generates the SAME seeded global array, keeps its
shard_range slice on its own GPU, calls reduce_multi, and checks the result
against the oracle of the whole array (bit-exact for int32 and min/max; G1 for
fp sums).  Uneven and empty shards are included.  Prints one JSON line per rank."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch
import torch.distributed as dist

import oracle
import synth
import paper_conf_cgo_gonzalohghmh19_b200 as rb


def main():
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    rank, world = dist.get_rank(), dist.get_world_size()
    comm = rb.Comm()

    def check_all(call):
        """call(t, op, mode) -> 1-element tensor; every dtype / size / op / mode
        against the oracle of the concatenated array."""
        fails, count = [], 0
        for dtype in ("int32", "float32", "float64"):
            for n in (0, 1, world - 1 if world > 1 else 0, 1000, (1 << 20) + 7, (1 << 24) + 3):
                x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", 7000 + n)
                lo, hi = rb.shard_range(n, world, rank)
                t = torch.empty(hi - lo + 1, dtype=getattr(torch, dtype), device=dev)[1:]
                if hi > lo:
                    t.copy_(torch.from_numpy(x[lo:hi]))
                for op in ("sum", "min", "max") + (("sum_accurate",) if dtype != "int32" else ()):
                    for mode in ("fast", "deterministic"):
                        got = call(t, op, mode).cpu().numpy()
                        ref = oracle.reduce(x, "sum" if op == "sum_accurate" else op)
                        count += 1
                        if dtype == "int32" or op not in ("sum", "sum_accurate"):
                            bits = int(got.view(np.uint32 if dtype != "float64" else np.uint64)[0])
                            if bits != ref.bits:
                                fails.append((dtype, n, op, mode, bits, ref.bits))
                        else:
                            ok, msg = oracle.check_sum(float(got[0]), ref, x.dtype, max(n, 1))
                            if not ok:
                                fails.append((dtype, n, op, mode, msg))
        return fails, count

    fails, count = check_all(lambda t, op, mode: rb.reduce_multi(t, op, comm, mode=mode))
    # the NVLS combine (reduce_multi_nvls): where the ranks share NVLink SHARP
    # multicast it must match the oracle like reduce_multi; elsewhere (one GPU)
    # creating it must fail cleanly with REDUCE_ERR_UNSUPPORTED on every rank
    # and leave the communicator usable
    nvls = {}
    for nv_mode in (1, 2):
        try:
            nv = rb.Nvls(comm, mode=nv_mode)
        except rb.ReduceError as e:
            nvls[nv_mode] = {"status": e.status, "error": str(e)[-300:]}
            continue
        f2, c2 = check_all(lambda t, op, mode: rb.reduce_multi_nvls(t, op, nv, mode=mode))
        torch.cuda.synchronize()
        dist.barrier()
        nv.destroy()
        nvls[nv_mode] = {"status": 0, "checked": c2, "fails": f2[:10]}
    after = rb.reduce_multi(torch.ones(1000, device=dev), "sum", comm).item()
    # deterministic mode: identical bits on every call
    x = synth.make("float32", (1 << 22) + 1, "uniform_pm1", 5)
    lo, hi = rb.shard_range(x.size, world, rank)
    t = torch.from_numpy(x[lo:hi]).to(dev)
    vals = {int(rb.reduce_multi(t, "sum", comm, mode="deterministic").cpu().view(torch.int32).item())
            for _ in range(20)}
    torch.cuda.synchronize()
    comm.destroy()
    dist.destroy_process_group()
    print(json.dumps({"rank": rank, "world": world, "checked": count, "fails": fails[:10],
                      "deterministic_distinct": len(vals), "nvls": nvls, "comm_after_nvls": after}), flush=True)


if __name__ == "__main__":
    main()
