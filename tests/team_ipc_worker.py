"""Worker for tests/test_team_gpu.py: two processes on the same GPU form a team
through CUDA IPC handles exchanged over a gloo process group, then run
reduce_multi_team on their shards and compare with the oracle."""
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
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)  # every member on the one GPU of the box (IPC within a device)
    team = rb.Team()
    fails, count = [], 0
    for dtype in ("int32", "float32", "float64"):
        for n in (7, 100000, (1 << 21) + 5):
            x = synth.make(dtype, n, "int_full" if dtype == "int32" else "uniform_pm1", 77 + n)
            lo, hi = rb.shard_range(n, world, rank)
            t = torch.from_numpy(np.ascontiguousarray(x[lo:hi])).cuda()
            for op in ("sum", "min", "max"):
                got = rb.reduce_multi_team(t, op, team).cpu().numpy()
                ref = oracle.reduce(x, op)
                count += 1
                if dtype == "int32" or op != "sum":
                    b = int(got.view(np.uint32 if dtype != "float64" else np.uint64)[0])
                    if b != ref.bits:
                        fails.append((dtype, n, op, b, ref.bits))
                else:
                    ok, msg = oracle.check_sum(float(got[0]), ref, x.dtype, n)
                    if not ok:
                        fails.append((dtype, n, op, msg))
    torch.cuda.synchronize()
    dist.barrier()
    team.destroy()
    dist.destroy_process_group()
    # one write(2) per line: the two workers share torchrun's stdout pipe
    os.write(1, (json.dumps({"rank": rank, "checked": count, "fails": fails[:5]}) + "\n").encode())


if __name__ == "__main__":
    main()
