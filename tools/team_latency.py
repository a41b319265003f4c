"""Cost of the cross-rank combine on one GPU (SURVEY 8(f) N2 vs S7).

Device time per call, from a CUDA graph of R back-to-back calls (cold inputs:
the calls rotate over a pool larger than L2 when the array is large), for
  reduce              single-GPU path (no combine)
  team k=1            reduce_multi_team: the exchange fused into the kernel epilogue
  nccl k=1            reduce_multi: raw partial + ncclAllReduce + finalize kernel
With one rank the exchange talks only to itself, so this isolates the fixed
overhead each combine adds to a call (fence, flags / collective launch); the
NVLink hop of a real multi-GPU team comes on top.
Run: python tools/team_latency.py  (one GPU; prints one JSON line per size)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torch.distributed as dist
    import paper_conf_cgo_gonzalohghmh19_b200 as rb

    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29541")
    os.environ.setdefault("RANK", "0")
    os.environ.setdefault("WORLD_SIZE", "1")
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("nccl", device_id=dev)
    team = rb.Team()
    comm = rb.Comm()
    stream = torch.cuda.Stream(dev)
    pool = torch.rand(1 << 29, device=dev)  # 2 GiB
    out = torch.empty(1, device=dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for lg in (10, 14, 18, 20, 22, 24, 26, 28):
        n = 1 << lg
        regions = max(1, min(64, pool.numel() // n))
        xs = [pool[i * n:(i + 1) * n] for i in range(regions)]
        R = max(8, min(200, (1 << 31) // (4 * n)))
        res = {"n": n}
        for name in ("reduce", "team_k1", "nccl_k1"):
            def call(x):
                if name == "reduce":
                    rb.reduce(x, "sum", out=out, stream=stream)
                elif name == "team_k1":
                    rb.reduce_multi_team(x, "sum", team, out=out, stream=stream)
                else:
                    rb.reduce_multi(x, "sum", comm, out=out, stream=stream)
            with torch.cuda.stream(stream):
                for i in range(3):
                    call(xs[i % regions])
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                for i in range(R):
                    call(xs[i % regions])
            best = 1e9
            for _ in range(3):
                with torch.cuda.stream(stream):
                    g.replay()
                    e0.record(stream)
                    g.replay()
                    e1.record(stream)
                torch.cuda.synchronize()
                best = min(best, e0.elapsed_time(e1) * 1e3 / R)
            res[name + "_us"] = round(best, 3)
            del g
        print(json.dumps(res), flush=True)
    torch.cuda.synchronize()
    team.destroy()
    comm.destroy()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
