#!/usr/bin/env python
"""Bench harness: device-wide reduction throughput on B200 (BASELINE.json metric
"reduction GB/s & fraction of HBM peak vs array size, 1/2/4/8 B200").

One step = one pass of the whole hot path (steps S0-S6, plus S7 for N>1) over
one batch of synthetic input already resident in HBM:
  N = 1 : reduce(fp32, sum) of n = 2^28 elements (1 GiB) -- the largest point
          of BASELINE configs[1] ("fp32 sum size sweep 1K-256M"), the headline.
  N > 1 : reduce_multi_team(fp32, sum): every rank reduces its own 2^28-element
          shard and the per-rank scalars meet in the kernel's epilogue over
          peer memory (--collective nccl: one NCCL all-reduce instead; the
          team path falls back to it if the peer mapping cannot be made).
          `value` is weak scaling (2^28 per GPU; at N = 8 this is the 8 GiB
          array of configs[4]); the same line carries `strong_scaling`: the
          fixed 2^31-element (8 GiB) array of configs[4], n_local = 2^31 / N
          per rank (`--scaling strong` makes it the `value`).
          The sharded result is checked against the sum of the per-rank local
          results once after warm-up, for every combine available
          (`cross_rank_check`).
`python bench.py --gpus N` without a torchrun environment re-executes itself
under torch.distributed.run with N ranks (one per GPU); under torchrun,
WORLD_SIZE must equal --gpus.
The 1 GiB per-GPU input is larger than the 126 MB L2, so consecutive steps
read from HBM without an explicit flush.

Extra keys: roofline (dominant kernel vs the measured HBM peak), cpu_baseline
(the oracle on the host cores), e2e (the same metric through the C-ABI host
entry with H2D/D2H copies in the timed region), clocks (NVML, sampled during
the timed region), gpu_launches, and `sweep` (fp32 sum GB/s vs size, each
call on a cold input region, with CUB's DeviceReduce and the CPU baseline --
oracle and OpenMP loop -- at the same n).

`--impl reference` times the CPU oracle (this tier's reference arm) on the
same config.  Launch: python bench.py --gpus N --steps K --warmup W
(N > 1 under torch.distributed.run, one rank per GPU).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_PER_GPU = 1 << 28
METRIC = "reduction GB/s & fraction of HBM peak vs array size, 1/2/4/8 B200"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", "--elements", dest="n", type=int, default=N_PER_GPU,
                    help="elements per GPU (spell it --elements under torchrun, whose parser eats --n)")
    ap.add_argument("--mode", default="fast", choices=["fast", "deterministic"])
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--sharded", action="store_true",
                    help="use the sharded path even at one rank (exercises S7 on one GPU)")
    ap.add_argument("--collective", default="team", choices=["team", "nccl", "nvls"],
                    help="cross-GPU combine: 'team' = fused into the reduction kernel over peer memory "
                         "(reduce_multi_team), 'nccl' = one ncclAllReduce of the per-rank scalar, 'nvls' = "
                         "fused into the kernel through NVLink SHARP multicast (reduce_multi_nvls: "
                         "multimem.ld_reduce in the NVSwitch)")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="which series is the line's `value`: weak = --elements per GPU, strong = "
                         "--strong-total elements split over the N GPUs (both are always reported)")
    ap.add_argument("--strong-total", type=int, default=1 << 31,
                    help="total elements of the strong-scaling array (default 2^31 = 8 GiB fp32, configs[4])")
    ap.add_argument("--nvls-check", action="store_true",
                    help="also build the NVLS combine (reduce_multi_nvls) and cross-check it (it is built anyway "
                         "with --collective nvls)")
    ap.add_argument("--share-gpu", action="store_true",
                    help="TEST MODE: every rank on cuda:0, gloo control plane, team combine over CUDA IPC "
                         "(validates the multi-rank path on a one-GPU box; timings are not scaling numbers)")
    return ap.parse_args()


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic():
    """dram bytes per launch of the dominant kernel from the committed ncu capture."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as f:
            s = json.load(f)
        return s.get("dram_bytes_per_launch"), s
    except Exception:
        return None, None


class ClockSampler:
    """NVML clocks + throttle reasons sampled in a thread during the timed region."""
    REASONS = {
        "sw_power_cap": 0x4, "hw_slowdown": 0x8, "sync_boost": 0x10, "sw_thermal_slowdown": 0x20,
        "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80, "applications_clocks_setting": 0x2,
    }

    def __init__(self, index: int):
        self.samples, self.mem_samples, self.reasons, self.ok = [], [], set(), False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # no NVML: report it, do not fake
            self.err = repr(e)
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.mem_samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_MEM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.001)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "")}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples),
                "mem_mhz": statistics.median(self.mem_samples) if self.mem_samples else None}


def gpu_identity(index: int):
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(index)
        name = pynvml.nvmlDeviceGetName(h)
        serial = pynvml.nvmlDeviceGetSerial(h)
        bus = pynvml.nvmlDeviceGetPciInfo(h).busId
        dec = lambda v: v.decode() if isinstance(v, bytes) else v
        return {"name": dec(name), "serial": dec(serial), "pci_bus": dec(bus)}
    except Exception as e:
        return {"error": repr(e)[:80]}


def software_env(dev):
    """GPU shape and software versions for the JSON line (metrics)."""
    import torch
    env = {}
    try:
        p = torch.cuda.get_device_properties(dev)
        env.update(sm_count=p.multi_processor_count, l2_bytes=getattr(p, "L2_cache_size", None),
                   hbm_bytes=p.total_memory, cc=f"{p.major}.{p.minor}")
    except Exception as e:
        env["device_error"] = repr(e)[:80]
    env["torch"] = torch.__version__
    env["cuda_runtime"] = torch.version.cuda
    try:
        env["nccl"] = ".".join(str(v) for v in torch.cuda.nccl.version())
    except Exception:
        pass
    try:
        import pynvml
        pynvml.nvmlInit()
        d = pynvml.nvmlSystemGetDriverVersion()
        env["driver"] = d.decode() if isinstance(d, bytes) else d
    except Exception:
        pass
    return env


def host_info():
    model = ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return model, len(os.sched_getaffinity(0))


def host_times(xh):
    """Median host time (us) of the oracle and of the OpenMP loop on xh (rank 0 context data)."""
    import oracle
    reps = 5 if xh.size <= (1 << 22) else 2
    outs = []
    for f in (lambda: oracle.reduce(xh, "sum"), lambda: oracle.omp_sum_f32(xh)):
        f()
        ts = []
        for _ in range(reps):
            t0 = time.perf_counter()
            f()
            ts.append(time.perf_counter() - t0)
        outs.append(round(statistics.median(ts) * 1e6, 2))
    return outs


# The paper's own numbers (speedup ratios only -- it reports no absolute
# throughput), quoted with their hardware: context, never a B200 target.
PAPER_CONTEXT = {
    "source": "Garcia De Gonzalo et al., CGO 2019 (PAPER.md); fp32, 64..2^28 elements, host<->device copies untimed "
              "(P:L463-L469, P:L641); baselines CUB 1.8.0 on the same GPU, OpenMP 4.0 on 2x8-core POWER8+",
    "hardware": {"Kepler": "K40c, nvcc 8.0.44", "Maxwell": "GTX980, nvcc 9.1.85", "Pascal": "P100, nvcc 9.2.88"},
    "claims": [
        {"where": "P:L601", "gpus": "K40c / GTX980 / P100", "sizes": "< 1M elements",
         "tangram_vs_cub": "2x-6x faster on average"},
        {"where": "P:L601", "gpus": "K40c / GTX980 / P100", "sizes": "> 1M elements",
         "tangram_vs_cub": "17%-38% slower (CUB's vector loads)"},
        {"where": "P:L685", "gpus": "Kepler K40c", "sizes": "1K-4M", "version": "(m)",
         "tangram_vs_cub": "4.6x", "tangram_vs_openmp": "3.6x"},
        {"where": "P:L687", "gpus": "Kepler K40c", "sizes": "> 4M", "tangram_vs_cub": "~38% slower"},
        {"where": "P:L733", "gpus": "Maxwell GTX980", "sizes": "65K-4M", "version": "(p)",
         "tangram_vs_cub": "4.6x", "tangram_vs_openmp": "3.4x"},
        {"where": "P:L735", "gpus": "Maxwell GTX980", "sizes": "> 4M", "tangram_vs_cub": "~7% slower"},
        {"where": "P:L777", "gpus": "Pascal P100", "sizes": "<= 1K", "tangram_vs_openmp": "on par"},
        {"where": "P:L777", "gpus": "Pascal P100", "sizes": "4K-65K", "tangram_vs_cub": "~8.5x",
         "tangram_vs_openmp": "~4.8x"},
        {"where": "P:L779", "gpus": "Pascal P100", "sizes": "65K-4M", "tangram_vs_cub": "4x"},
        {"where": "P:L781", "gpus": "Pascal P100", "sizes": "> 4M", "tangram_vs_cub": "27% slower"},
    ],
}


def paper_context(sweep):
    """PAPER_CONTEXT plus this run's like-for-like ratios on the B200: the
    library vs CUB 12.9's DeviceReduce on the same device, per size class of
    the paper (geometric mean over the fp32 U[0,1) sweep points in the class)."""
    ctx = dict(PAPER_CONTEXT)
    if not sweep:
        return ctx
    classes = (("< 1M elements", 0, 1 << 20), ("1K-4M", 1 << 10, 1 << 22), ("65K-4M", 1 << 16, 1 << 22),
               ("4K-65K", 1 << 12, 1 << 16), ("> 1M elements", (1 << 20) + 1, 1 << 40), ("> 4M", (1 << 22) + 1, 1 << 40))
    b200 = {}
    for name, lo, hi in classes:
        r = [e["speedup_vs_cub"] for e in sweep if e.get("dist") == "U[0,1)" and lo <= e["n"] <= hi
             and e.get("speedup_vs_cub")]
        if r:
            g = 1.0
            for v in r:
                g *= v
            b200[name] = {"ours_vs_cub_geomean": round(g ** (1 / len(r)), 3), "points": len(r)}
    ctx["b200_this_run"] = b200
    ctx["note"] = ("the paper's gains over CUB 1.8 came from CUB's small-array overheads on Kepler-Pascal; "
                   "CUB in CUDA 12.9 on B200 has none of them, so like-for-like ratios here are smaller")
    return ctx


# --------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """This tier's reference arm: the CPU oracle, as it stands, on the host cores."""
    if rank != 0:
        return
    import numpy as np
    import oracle
    import synth
    n = args.n
    # bounded sample of the workload so (W + K) steps finish in about a minute
    probe = synth.make("float32", 1 << 22, "uniform01", 1)
    t0 = time.perf_counter(); oracle.reduce(probe, "sum"); t1 = time.perf_counter()
    rate = (1 << 22) / max(t1 - t0, 1e-6)
    budget_s = 60.0
    sample_n = int(min(n, max(1 << 20, rate * budget_s / max(1, args.steps + args.warmup))))
    sample_n -= sample_n % 8
    x = synth.make("float32", sample_n, "uniform01", synth.seed_for(1, n))
    for _ in range(args.warmup):
        oracle.reduce(x, "sum")
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.reduce(x, "sum")
    dt = (time.perf_counter() - t0) / args.steps
    gbs = sample_n * 4 / dt / 1e9
    model, cores = host_info()
    line = {
        "impl": "reference", "metric": METRIC, "value": round(gbs, 4), "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 4),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": workload_config(args, world, None),
        "cpu_baseline": {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": f"first {sample_n} elements of the seeded 2^28 fp32 U[0,1) workload per step "
                                   f"(Neumaier sum in double, oracle/oracle.c), host {model}"},
        "e2e": {"value": round(gbs, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(args, world, plan, sharded=False):
    cfg = {"workload": f"fp32 sum of {args.n} (2^{args.n.bit_length() - 1}) elements per GPU"
                       + (" -- BASELINE configs[1] largest point" if world == 1 else
                          f" -- BASELINE configs[4] sharded sum, {world} GPUs, per-rank partials combined "
                          + {"team": "in the reduction kernel over peer memory (reduce_multi_team)",
                             "nvls": "in the reduction kernel through NVLS multicast (reduce_multi_nvls)",
                             "nccl": "by one NCCL all-reduce"}[args.collective]),
           "n_per_gpu": args.n, "total_bytes": args.n * 4 * world, "op": "sum", "mode": args.mode,
           "parallelism": f"shard{world}" if (world > 1 or sharded) else "single-gpu",
           "collective": args.collective if (world > 1 or sharded) else None,
           "l2": "inputs (4 B x n per GPU) larger than the 126 MB L2 between steps; no flush needed",
           "distribution": "U[0,1) fp32, numpy PCG64 seed 2019+1000*1+log2(n)+rank"}
    if plan is not None:
        cfg["variant"] = plan
    return cfg


def spawn_or_check_world(args):
    """One process per GPU.  `--gpus N` (N > 1) outside torchrun re-executes this
    script under torch.distributed.run with N ranks and exits with its status;
    under torchrun, WORLD_SIZE must equal --gpus (else exit 2: a bench line
    must never claim N GPUs while timing a different number of ranks)."""
    ws = os.environ.get("WORLD_SIZE")
    if ws is None:
        if args.gpus > 1 and args.impl == "ours":
            import socket
            import subprocess
            with socket.socket() as sk:
                sk.bind(("127.0.0.1", 0))
                port = sk.getsockname()[1]
            cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
                   "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
            print(f"bench: spawning {args.gpus} ranks: {' '.join(cmd)}", file=sys.stderr, flush=True)
            sys.exit(subprocess.run(cmd).returncode)
        return
    if int(ws) != args.gpus:
        print(f"bench: WORLD_SIZE={ws} but --gpus {args.gpus}: refusing to time a different rank count",
              file=sys.stderr, flush=True)
        sys.exit(2)


# --------------------------------------------------------------- our arm
def main():
    args = parse()
    spawn_or_check_world(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world if "WORLD_SIZE" in os.environ else args.gpus)

    import numpy as np
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_cgo_gonzalohghmh19_b200 as rb

    if args.share_gpu and args.collective != "team":
        raise SystemExit("--share-gpu needs --collective team (NCCL refuses two ranks on one GPU)")
    local = 0 if args.share_gpu else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    sharded = world > 1 or args.sharded
    if sharded:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        os.environ.setdefault("RANK", str(rank))
        os.environ.setdefault("WORLD_SIZE", str(world))
        if args.share_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    def allmax(v):
        """max over ranks of a host float (device tensor for NCCL, host for gloo)"""
        if world == 1 and not sharded:
            return v
        t = torch.tensor([v], dtype=torch.float64, device="cpu" if args.share_gpu else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    n = args.n
    x_host = synth.make("float32", n, "uniform01", synth.seed_for(1, n, rank))
    x = torch.from_numpy(x_host).to(dev)
    out = torch.empty(1, dtype=torch.float32, device=dev)
    stream = torch.cuda.Stream(dev)
    comm = None
    collective_note = None
    combines = {}  # name -> Team / Comm of every cross-GPU combine this run could build
    comm_info = None
    if sharded:
        try:
            combines["team"] = rb.Team()
        except rb.ReduceError as e:  # e.g. no peer mapping between the GPUs
            if args.share_gpu:
                raise
            combines["team"] = None
            collective_note = f"team combine unavailable ({e})"
        nvls_note = None
        if args.share_gpu:
            combines["nccl"] = None  # NCCL refuses two ranks on one GPU
            combines["nvls"] = None
            nvls_note = "ranks share one GPU"
        else:
            combines["nccl"] = rb.Comm()
            if args.collective == "nvls" or args.nvls_check:
                try:  # a collective: every rank gets the same outcome
                    combines["nvls"] = rb.Nvls(combines["nccl"], mode=1)
                except rb.ReduceError as e:
                    combines["nvls"] = None
                    nvls_note = str(e)[-200:]
            else:
                combines["nvls"] = None
                nvls_note = "not requested (--collective nvls or --nvls-check)"
        if combines.get(args.collective) is None:
            if args.collective in ("team", "nvls") and combines.get("nccl") is not None:
                collective_note = ((collective_note or f"{args.collective} combine unavailable")
                                   + (f" ({nvls_note})" if args.collective == "nvls" else "")
                                   + "; fell back to the NCCL all-reduce")
                print(f"bench: {collective_note}", file=sys.stderr)
                args.collective = "nccl"
            else:
                raise SystemExit(f"bench: the {args.collective} combine is unavailable")
        comm = combines[args.collective]
        comm_info = {"world_size": world,
                     "team_members": None if combines.get("team") is None else combines["team"].world,
                     "nccl_comm_nranks": None if combines.get("nccl") is None else combines["nccl"].nranks(),
                     "nvls": "available" if combines.get("nvls") is not None else f"unavailable: {nvls_note}",
                     "process_group_backend": dist.get_backend()}
        if comm_info["nccl_comm_nranks"] not in (None, world) or comm_info["team_members"] not in (None, world):
            raise SystemExit(f"bench: communicator size disagrees with WORLD_SIZE: {comm_info}")
    plan = rb.query_plan("float32", "sum", n, in_ptr=x.data_ptr(), mode=args.mode)
    rb.prepare(stream, n)

    def sharded_call(name, xt, o):
        if name == "team":
            rb.reduce_multi_team(xt, "sum", combines["team"], out=o, stream=stream, mode=args.mode)
        elif name == "nvls":
            rb.reduce_multi_nvls(xt, "sum", combines["nvls"], out=o, stream=stream, mode=args.mode)
        else:
            rb.reduce_multi(xt, "sum", combines["nccl"], out=o, stream=stream, mode=args.mode)

    def step():
        if comm is None:
            rb.reduce(x, "sum", out=out, stream=stream, mode=args.mode)
        else:
            sharded_call(args.collective, x, out)

    def sync_all():
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    def cross_rank_check(name, xt):
        """The sharded result of combine `name` against the per-rank local
        results summed over the torch process group (an independent path): the
        relative gap must be at the fp32 rounding level of the final conversions."""
        o = torch.empty(1, dtype=torch.float32, device=dev)
        loc = torch.empty(1, dtype=torch.float32, device=dev)
        with torch.cuda.stream(stream):
            sharded_call(name, xt, o)
            rb.reduce(xt, "sum", out=loc, stream=stream, mode=args.mode)
        torch.cuda.synchronize(dev)
        got = float(o.item())
        t = torch.tensor([float(loc.item())], dtype=torch.float64, device="cpu" if args.share_gpu else dev)
        dist.all_reduce(t)
        want = float(t.item())
        rel = abs(got - want) / max(abs(want), 1e-30)
        # every rank must agree on the bits as well (the combine is one value for all)
        g = torch.tensor([got], dtype=torch.float64, device="cpu" if args.share_gpu else dev)
        gmax, gmin = g.clone(), g.clone()
        dist.all_reduce(gmax, op=dist.ReduceOp.MAX)
        dist.all_reduce(gmin, op=dist.ReduceOp.MIN)
        res = {"sharded": got, "sum_of_local": want, "rel_gap": rel, "ranks_agree": float(gmax) == float(gmin),
               "ok": rel <= 4 * world * 2.0 ** -24 and float(gmax) == float(gmin)}
        if not res["ok"]:
            print(f"bench: {name} sharded result check failed: {res}", file=sys.stderr)
        return res

    with torch.cuda.stream(stream):
        for _ in range(max(3, args.warmup)):
            step()
    sync_all()
    cross_check = None
    if comm is not None:
        cross_check = {}
        for name in ("team", "nccl", "nvls"):
            cross_check[name] = (cross_rank_check(name, x) if combines.get(name) is not None
                                 else "unavailable" + (" (ranks share one GPU)" if args.share_gpu and name != "team"
                                                       else (f" ({nvls_note})" if name == "nvls" else "")))
        sync_all()
    # Single GPU: the K steps are captured once into a CUDA graph and replayed
    # (no host launch gaps between steps; the same kernels on the same
    # HBM-resident input).  The plain stream-launched loop is timed as well.
    graph = None
    if comm is None:
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=stream):
            for _ in range(args.steps):
                step()
        with torch.cuda.stream(stream):
            graph.replay()  # warm the graph once
        sync_all()
    # ---- timed region: K steps between two events on the launch stream
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clocks = ClockSampler(local)
    with clocks:
        with torch.cuda.stream(stream):
            e0.record(stream)
            if graph is not None:
                graph.replay()
            else:
                for _ in range(args.steps):
                    step()
            e1.record(stream)
        e1.synchronize()
    sync_all()
    ms = e0.elapsed_time(e1) / args.steps
    if world > 1:
        ms = allmax(ms)
    value = world * n * 4 / (ms * 1e-3) / 1e9

    # ---- strong scaling: the fixed --strong-total array
    # (2^31 fp32 = 8 GiB, configs[4]) split into contiguous shards, rank r owns
    # [floor(r T / N), floor((r+1) T / N)) drawn on its own GPU; K steps of the
    # same path (graph-replayed at N = 1, stream-launched sharded calls at N > 1).
    strong = None
    strong_clocks = None
    if args.strong_total > 0:
        lo_s, hi_s = rb.shard_range(args.strong_total, world, rank)
        n_s = hi_s - lo_s
        gen = torch.Generator(device=dev).manual_seed(2019 + 1000 * 4 + 31 + rank)
        xs = torch.rand(n_s, dtype=torch.float32, device=dev, generator=gen)
        os_ = torch.empty(1, dtype=torch.float32, device=dev)
        rb.prepare(stream, n_s)

        def sstep():
            if comm is None:
                rb.reduce(xs, "sum", out=os_, stream=stream, mode=args.mode)
            else:
                sharded_call(args.collective, xs, os_)
        with torch.cuda.stream(stream):
            for _ in range(max(3, args.warmup)):
                sstep()
        sync_all()
        s_check = cross_rank_check(args.collective, xs) if comm is not None else None
        sync_all()
        sgraph = None
        if comm is None:
            sgraph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(sgraph, stream=stream):
                for _ in range(args.steps):
                    sstep()
            with torch.cuda.stream(stream):
                sgraph.replay()
            sync_all()
        strong_clocks = ClockSampler(local)
        with strong_clocks:
            with torch.cuda.stream(stream):
                e0.record(stream)
                if sgraph is not None:
                    sgraph.replay()
                else:
                    for _ in range(args.steps):
                        sstep()
                e1.record(stream)
            e1.synchronize()
        sync_all()
        s_ms = allmax(e0.elapsed_time(e1) / args.steps) if world > 1 else e0.elapsed_time(e1) / args.steps
        strong = {"total_elements": args.strong_total, "total_bytes": args.strong_total * 4,
                  "n_local_rank0": rb.shard_range(args.strong_total, world, 0)[1], "ms_per_step": round(s_ms, 5),
                  "value": round(args.strong_total * 4 / (s_ms * 1e-3) / 1e9, 2), "unit": "GB/s",
                  "elements_per_s": round(args.strong_total / (s_ms * 1e-3), 1),
                  "launch": "cuda-graph replay" if sgraph is not None else f"stream (sharded, {args.collective})",
                  "data": "torch.rand U[0,1) fp32 on each rank's own GPU, seed 2019+4031+rank",
                  "clocks": strong_clocks.summary()}
        if s_check is not None:
            strong["cross_rank_check"] = s_check
        del sgraph, xs
        torch.cuda.empty_cache()
    # sharded: the same K steps without the cross-rank combine (local reduce
    # only), so the combine's cost per step is visible
    decomposition = None
    if comm is not None:
        sync_all()
        with torch.cuda.stream(stream):
            e0.record(stream)
            for _ in range(args.steps):
                rb.reduce(x, "sum", out=out, stream=stream, mode=args.mode)
            e1.record(stream)
        e1.synchronize()
        local_ms = allmax(e0.elapsed_time(e1) / args.steps)
        sync_all()
        decomposition = {"local_reduce_ms_per_step": round(local_ms, 5),
                         "combine_us_per_step": round((ms - local_ms) * 1e3, 3),
                         "how": "max over ranks of K stream-launched local reduce() calls vs the K sharded calls"}
    stream_ms = None
    if graph is not None:  # the same K steps launched one by one from the host
        with torch.cuda.stream(stream):
            e0.record(stream)
            for _ in range(args.steps):
                step()
            e1.record(stream)
        e1.synchronize()
        stream_ms = e0.elapsed_time(e1) / args.steps
        del graph

    # ---- dominant kernel: k_reduce.  At N = 1 a step is exactly one k_reduce
    # launch (plan.launches == 1), so its average launch duration is the timed
    # region / K; event pairs around single launches are reported alongside
    # (they include each launch's ramp-up / drain).
    kern_ms = []
    with torch.cuda.stream(stream):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(50)]
        for a, b in evs:
            a.record(stream)
            rb.reduce(x, "sum", out=out, stream=stream, mode=args.mode)
            b.record(stream)
    torch.cuda.synchronize(dev)
    kern_ms = [a.elapsed_time(b) for a, b in evs]
    k_event = statistics.mean(kern_ms)
    kavg = ms if (comm is None and plan["launches"] == 1) else k_event
    peak, peak_src = measured_peaks()
    achieved = n * 4 / (kavg * 1e-3) / 1e9
    # the same copy the driver's MEASURED_PEAKS uses (b.copy_(a), 1 Gi bf16,
    # read + write bytes, best of 10), on THIS box: B200s in the pool differ
    copy_gbs = None
    try:
        ca = torch.empty(1 << 30, dtype=torch.bfloat16, device=dev)
        cb = torch.empty_like(ca)
        cb.copy_(ca)
        best_ms = None
        for _ in range(10):
            ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ea.record()
            cb.copy_(ca)
            eb.record()
            eb.synchronize()
            t = ea.elapsed_time(eb)
            best_ms = t if best_ms is None else min(best_ms, t)
        copy_gbs = round(2 * ca.numel() * 2 / (best_ms * 1e-3) / 1e9, 1)
        del ca, cb
        torch.cuda.empty_cache()
    except Exception:
        pass
    traffic, ncu_s = ncu_traffic()
    roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic,
                "kernel": "rb::k_reduce<f32,sum,U,Vs,stage> (+ grid combine epilogue)",
                "algorithmic_bytes_per_launch": n * 4, "avg_launch_ms": round(kavg, 5),
                "single_launch_event_ms": round(k_event, 5),
                "peak_source": peak_src, "frac_of_nominal_8TBps": round(achieved / 8000.0, 4),
                "same_box_copy_gbs": copy_gbs,
                "frac_of_same_box_copy": None if not copy_gbs else round(achieved / copy_gbs, 4)}
    # kernel share of the step (compare with the committed ncu launch list)
    roofline["kernel_share_of_step"] = round(min(1.0, kavg / ms), 4)

    # ---- e2e through the C-ABI host entry (H2D + reduce + D2H in the timed region)
    e2e = None
    if not args.no_e2e:
        pinned = torch.from_numpy(x_host).pin_memory()
        k_e2e = max(3, min(args.steps, 20))
        if comm is None:
            rb.reduce_host(pinned, "sum", stream=stream, mode=args.mode)
            sync_all()
            t0 = time.perf_counter()
            for _ in range(k_e2e):
                rb.reduce_host(pinned, "sum", stream=stream, mode=args.mode)
            dt = (time.perf_counter() - t0) / k_e2e
        else:
            xd = torch.empty_like(x)
            sync_all()
            t0 = time.perf_counter()
            with torch.cuda.stream(stream):
                for _ in range(k_e2e):
                    xd.copy_(pinned, non_blocking=True)
                    sharded_call(args.collective, xd, out)
                    out.item()
            dt = allmax((time.perf_counter() - t0) / k_e2e)
        # the PCIe ceiling e2e runs against: a plain pinned H2D copy of the same bytes
        h2d_gbs = None
        try:
            xd2 = torch.empty_like(x)
            best = None
            for _ in range(3):
                ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                with torch.cuda.stream(stream):
                    ea.record(stream)
                    xd2.copy_(pinned, non_blocking=True)
                    eb.record(stream)
                eb.synchronize()
                best = ea.elapsed_time(eb) if best is None else min(best, ea.elapsed_time(eb))
            h2d_gbs = round(n * 4 / (best * 1e-3) / 1e9, 2)
            del xd2
        except Exception:
            pass
        e2e = {"value": round(world * n * 4 / dt / 1e9, 3), "unit": "GB/s", "h2d_bytes_per_step": n * 4,
               "h2d_copy_only_gbs": h2d_gbs,
               "d2h_bytes_per_step": 4, "ms_per_step": round(dt * 1e3, 3),
               "path": "reduce_host (C ABI, pinned host buffer, chunked H2D overlapped with the chunk reductions)"
               if comm is None else f"pinned H2D copy + reduce_multi ({args.collective}) + D2H of the result"}

    # ---- size sweep (N = 1): device time per call from a CUDA graph of R calls
    # over disjoint, never-recently-touched regions of the resident 1 GiB input
    # (cold: every call reads HBM), plus the small-array latency regime
    # (BASELINE configs[3]) measured three ways.
    sweep = latency = None
    if not args.no_sweep and world == 1:
        sys.path.insert(0, os.path.join(ROOT, "tools"))
        from cudatiming import time_calls, disjoint_regions
        try:
            from tests import cub as cubref
            cubref.lib()
        except Exception:
            cubref = None
        outs = torch.empty(4096, dtype=torch.float32, device=dev)
        # C2: every power of two 2^10..2^28 elements, U[0,1) and
        # U[-1,1).  Columns: cold (each call of the graph reads a region nobody
        # touched recently: HBM) with the default stream ordering; cold with
        # REDUCE_FLAG_INPUT_READY (inputs written long before: early register
        # loads allowed); L2-warm (the same region every call; above the 126 MB
        # L2 it is HBM again); CUB's DeviceReduce on the cold regions.
        x_pm1 = (x * 2 - 1).contiguous()
        sweep = []
        for dist_name, pool in (("U[0,1)", x), ("U[-1,1)", x_pm1)):
            for k in range(10, 29):
                m = 1 << k
                # >= 20 calls per graph (the graph's own launch latency, ~1-3 us, is
                # spread over R calls); regions cycle only when each is far beyond
                # what L2 can keep between revisits (disjoint_regions)
                R = max(20, min(100, (256 << 20) // (4 * m)))
                warm, timed = disjoint_regions(pool, R, m)
                p = rb.query_plan("float32", "sum", m, in_ptr=timed[0].data_ptr(), mode=args.mode)
                ctr = [0]

                def launch(t, **kw):
                    ctr[0] = (ctr[0] + 1) % 4096
                    rb.reduce(t, "sum", out=outs[ctr[0]:ctr[0] + 1], stream=stream, mode=args.mode, **kw)
                sec = time_calls(launch, warm, timed, stream, repeats=3)
                sec_ready = time_calls(lambda t: launch(t, input_ready=True), warm, timed, stream, repeats=3)
                sec_warm = time_calls(launch, [timed[0]] * R, [timed[0]] * R, stream, repeats=3)
                gbs = m * 4 / sec / 1e9
                cub_sec = None
                if cubref is not None:  # the paper's comparison system, on the same device (context)
                    def launch_cub(t):
                        ctr[0] = (ctr[0] + 1) % 4096
                        cubref.reduce(1, 0, t.data_ptr(), t.numel(), outs[ctr[0]:ctr[0] + 1].data_ptr(),
                                      stream.cuda_stream)
                    cubref.reduce(1, 0, timed[0].data_ptr(), m, outs.data_ptr(), stream.cuda_stream)  # temp storage
                    torch.cuda.synchronize(dev)
                    cub_sec = time_calls(launch_cub, warm, timed, stream, repeats=3)
                row = {"dist": dist_name, "n": m, "log2_n": k, "paper_size_point": k % 2 == 0,
                       "us": round(sec * 1e6, 3), "GBps": round(gbs, 1),
                       "elements_per_s": round(m / sec, 1), "frac_of_peak": round(gbs / peak, 4),
                       "frac_of_nominal_8TBps": round(gbs / 8000.0, 4),
                       "input_ready_us": round(sec_ready * 1e6, 3),
                       "input_ready_GBps": round(m * 4 / sec_ready / 1e9, 1),
                       "l2_warm_us": round(sec_warm * 1e6, 3),
                       "l2_warm_GBps": round(m * 4 / sec_warm / 1e9, 1),
                       "cub_us": None if cub_sec is None else round(cub_sec * 1e6, 3),
                       "speedup_vs_cub": None if cub_sec is None else round(cub_sec / sec, 3),
                       "variant": f"gc{p['grid_combine']} g{p['grid']}x{p['block']} u{p['unroll']}"}
                if dist_name == "U[0,1)":
                    # the CPU beside it at the same n (the paper's CPU
                    # crossover): the oracle (1 thread) and the OpenMP pragma loop
                    row["cpu_oracle_us"], row["cpu_omp_us"] = host_times(x_host[:m])
                sweep.append(row)
        del x_pm1
        latency = []
        for dt in ("int32", "float32"):
            tdt = getattr(torch, dt)
            src = torch.ones(1 << 20, dtype=tdt, device=dev)
            o1 = torch.empty(4096, dtype=tdt, device=dev)
            for m in (32, 1024, 65536):
                warm, timed = disjoint_regions(src, 50, m)
                ctr = [0]

                def launch(t, o1=o1):
                    ctr[0] = (ctr[0] + 1) % 4096
                    rb.reduce(t, "sum", out=o1[ctr[0]:ctr[0] + 1], stream=stream)
                g_us = time_calls(launch, warm, timed, stream, repeats=3) * 1e6
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                for t in timed:
                    launch(t)
                b.record(stream)
                b.synchronize()
                s_us = a.elapsed_time(b) * 1e3 / len(timed)
                walls = []
                for t in timed[:20]:
                    t0 = time.perf_counter()
                    launch(t)
                    stream.synchronize()
                    walls.append(time.perf_counter() - t0)
                latency.append({"dtype": dt, "n": m, "graph_us": round(g_us, 3), "stream_b2b_us": round(s_us, 3),
                                "host_wall_us": round(statistics.median(walls) * 1e6, 2)})

    # ---- every (dtype, op) at 1 GiB (the resident input reinterpreted; > L2):
    # device time per call from a graph of 20 calls, default dispatch.
    ops_1gib = None
    if not args.no_sweep and world == 1:
        ops_1gib = []
        for dt_name, tdt in (("int32", torch.int32), ("float32", torch.float32), ("float64", torch.float64)):
            xv = x.view(tdt)
            for op in ("sum", "min", "max") + (("sum_accurate",) if dt_name != "int32" else ()):
                o1 = torch.empty(1, dtype=tdt, device=dev)

                def launch_o(t, op=op, o1=o1):
                    rb.reduce(t, op, out=o1, stream=stream, mode=args.mode)
                sec = time_calls(launch_o, [xv] * 3, [xv] * 20, stream, repeats=2)
                pp = rb.query_plan(dt_name, op, xv.numel(), in_ptr=xv.data_ptr(), mode=args.mode)
                ops_1gib.append({"dtype": dt_name, "op": op, "us": round(sec * 1e6, 2),
                                 "GBps": round(n * 4 / sec / 1e9, 1), "frac_of_peak": round(n * 4 / sec / 1e9 / peak, 4),
                                 "variant": f"gc{pp['grid_combine']} g{pp['grid']}x{pp['block']} u{pp['unroll']} st{pp['stage']}"})

    # ---- BASELINE configs[0]: int32 sum of 1 M full-range elements vs the CPU
    # oracle (bit-exact) -- device time per call, and the oracle on the host
    cfg1 = cfg3 = None
    if not args.no_sweep and world == 1:
        import oracle
        m = 1 << 20
        oi = torch.empty(4096, dtype=torch.int32, device=dev)
        cfg1 = []
        # C1: full-range values (every block's sum wraps) and the
        # small range randint(-1000, 1001), each in both modes; device time per
        # call from a graph over cold regions holding that very distribution,
        # the bit-exact check of one call on the seeded array, and the oracle.
        for dist_i in ("int_full", "int_small"):
            xi_h = synth.make("int32", m, dist_i, synth.seed_for(0, m))
            xi = torch.from_numpy(xi_h).to(dev)
            pool_i = xi.repeat(64)  # 64 cold-able copies (256 MB > L2)
            warm_i, timed_i = disjoint_regions(pool_i, 32, m)
            t0 = time.perf_counter()
            want = int(oracle.reduce(xi_h, "sum").value)
            cpu_us = (time.perf_counter() - t0) * 1e6
            for mode_i in ("fast", "deterministic"):
                ctr = [0]

                def launch_i(t, mode_i=mode_i):
                    ctr[0] = (ctr[0] + 1) % 4096
                    rb.reduce(t, "sum", out=oi[ctr[0]:ctr[0] + 1], stream=stream, mode=mode_i)
                gpu_us = time_calls(launch_i, warm_i, timed_i, stream, repeats=3) * 1e6
                got = int(rb.reduce(xi, "sum", stream=stream, mode=mode_i).cpu().item())
                pp = rb.query_plan("int32", "sum", m, in_ptr=xi.data_ptr(), mode=mode_i)
                cfg1.append({"n": m, "dist": dist_i, "mode": mode_i, "gpu_us": round(gpu_us, 3),
                             "GBps": round(m * 4 / gpu_us / 1e3, 1), "cpu_oracle_us": round(cpu_us, 1),
                             "bit_exact": got == want,
                             "variant": f"gc{pp['grid_combine']} g{pp['grid']}x{pp['block']} u{pp['unroll']}"})
            del pool_i
        # ---- BASELINE configs[2]: int32 / fp64 sum, min, max at 64 M elements,
        # atomic (fast) vs deterministic-tree grid combine
        cfg3 = []
        for dt_name, tdt, es in (("int32", torch.int32, 4), ("float64", torch.float64, 8)):
            m = 1 << 26
            regs_w, regs_t = disjoint_regions(x.view(tdt), 4, m)
            o3 = torch.empty(4096, dtype=tdt, device=dev)
            for op in ("sum", "min", "max"):
                row = {"dtype": dt_name, "op": op, "n": m}
                # atomic = "DT,A" (red.global per block + ticket), tree = strict
                # deterministic (partials + k_combine), auto = the table's fast-mode pick
                arms = (("atomic", dict(grid_combine=1)), ("tree", dict(mode="deterministic", grid_combine=2)),
                        ("auto_fast", dict()), ("auto_deterministic", dict(mode="deterministic")))
                for arm, kw in arms:
                    def launch_3(t, op=op, kw=kw, o3=o3):
                        ctr[0] = (ctr[0] + 1) % 4096
                        rb.reduce(t, op, out=o3[ctr[0]:ctr[0] + 1], stream=stream, **kw)
                    sec = time_calls(launch_3, regs_w, regs_t, stream, repeats=2)
                    pp = rb.query_plan(dt_name, op, m, in_ptr=regs_t[0].data_ptr(), **kw)
                    row[arm] = {"us": round(sec * 1e6, 2), "GBps": round(m * es / sec / 1e9, 1),
                                "grid_combine": rb.GC_NAMES[pp["grid_combine"]],
                                "grid": pp["grid"], "block": pp["block"], "unroll": pp["unroll"]}
                if dt_name == "float64" and op == "sum":
                    # distinct results over 20 runs on the same input
                    for arm, kw in (("atomic", dict(grid_combine=1)), ("tree", dict(mode="deterministic", grid_combine=2))):
                        outs20 = torch.empty(20, dtype=tdt, device=dev)
                        for i in range(20):
                            rb.reduce(regs_t[0], op, out=outs20[i:i + 1], stream=stream, **kw)
                        torch.cuda.synchronize(dev)
                        row[arm]["distinct_results_20_runs"] = len(set(outs20.cpu().numpy().tobytes()[8 * i:8 * i + 8]
                                                                        for i in range(20)))
                cfg3.append(row)

    # ---- BASELINE configs[4] at k = 1: one 8 GiB (2^31 fp32) array on one GPU
    # (64-bit indexing) is the strong-scaling series' N = 1 point (above); its
    # parity is tests/test_parity_gpu.py's full-size test.
    big = strong if world == 1 else None

    # ---- histogram of the resident 1 GiB, 256 and 65536 bins
    hist = None
    if not args.no_sweep and world == 1:
        hist = []
        for nbins in (256, 65536):
            hc = torch.empty(nbins, dtype=torch.int32, device=dev)

            def launch_h(t, hc=hc, nbins=nbins):
                rb.histogram(t, 0.0, 1.0, nbins, counts=hc, stream=stream)
            sec = time_calls(launch_h, [x] * 2, [x] * 10, stream, repeats=2)
            hist.append({"dtype": "float32", "n": n, "nbins": nbins, "us": round(sec * 1e6, 2),
                         "GBps": round(n * 4 / sec / 1e9, 1)})

    # ---- many small arrays in one launch: batched rows of
    # the resident input, device time per call (graph), against one reduce()
    # per array (the sweep's per-call time at that length).
    batched = None
    if not args.no_sweep and world == 1:
        batched = []
        per_call = {e["n"]: e["us"] for e in sweep if e["dist"] == "U[0,1)"}
        for cols in (64, 1024, 16384):
            rows = (256 << 20) // (4 * cols)
            xv = x[: rows * cols].view(rows, cols)
            ob = torch.empty(rows, dtype=torch.float32, device=dev)

            def launch_b(t, ob=ob, xv=xv):
                rb.reduce_batched(xv, "sum", out=ob, stream=stream)
            sec = time_calls(launch_b, [xv] * 3, [xv] * 10, stream, repeats=2)
            one = per_call.get(cols)
            batched.append({"rows": rows, "cols": cols, "us": round(sec * 1e6, 2),
                            "GBps": round(rows * cols * 4 / sec / 1e9, 1),
                            "arrays_per_s": round(rows / sec, 1),
                            "speedup_vs_one_reduce_per_array": None if one is None else round(one * 1e-6 * rows / sec, 1)})

    # ---- variable-length segments through an offsets array (N1, the
    # element-balanced chunk kernels): 256 MB of the resident input cut into
    # power-law (mean 64) and uniform (0..128, 0..2048) lengths, seeded
    segmented = None
    if not args.no_sweep and world == 1:
        segmented = []
        rng_s = np.random.Generator(np.random.PCG64(2019 + 1000 * 6))
        total = (256 << 20) // 4
        for dist_s, mean in (("powerlaw", 64), ("uniform", 64), ("uniform", 1024)):
            nseg = total // mean
            if dist_s == "uniform":
                lens = rng_s.integers(0, 2 * mean + 1, nseg)
            else:
                lens = np.minimum((rng_s.pareto(1.2, nseg) * mean * 0.2).astype(np.int64) + 1, 1 << 20)
            offs = np.minimum(np.concatenate([[0], np.cumsum(lens)]), total)
            ot = torch.from_numpy(offs).to(dev)
            xs = x[: int(offs[-1])]
            ob = torch.empty(nseg, dtype=torch.float32, device=dev)

            def launch_s(t, ob=ob, xs=xs, ot=ot):
                rb.reduce_segmented(xs, ot, "sum", out=ob, stream=stream)
            sec = time_calls(launch_s, [xs] * 3, [xs] * 10, stream, repeats=2)
            segmented.append({"lengths": f"{dist_s} mean {mean}", "segments": nseg, "elements": int(offs[-1]),
                              "us": round(sec * 1e6, 2), "GBps": round(int(offs[-1]) * 4 / sec / 1e9, 1),
                              "segments_per_s": round(nseg / sec, 1)})

    # ---- CPU baseline: the oracle on the host cores (rank 0, N = 1)
    cpu = None
    if not args.no_cpu and world == 1 and rank == 0:
        import oracle
        model, ncores = host_info()
        reps = 2
        oracle.reduce(x_host[: 1 << 20], "sum")
        t0 = time.perf_counter()
        for _ in range(reps):
            oracle.reduce(x_host, "sum")
        dt = (time.perf_counter() - t0) / reps
        cpu = {"value": round(n * 4 / dt / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"the full 2^28-element fp32 workload, {reps} repetitions (Neumaier in double, "
                         f"single thread) on {model} ({ncores} usable cores)"}
        t0 = time.perf_counter()
        for _ in range(reps):
            oracle.omp_sum_f32(x_host)
        dto = (time.perf_counter() - t0) / reps
        cpu_omp = {"value": round(n * 4 / dto / 1e9, 3), "unit": "GB/s", "cores": oracle.omp_threads(),
                   "kind": "paper-style OpenMP reduce pragma (P:L469), context only"}

    if rank == 0:
        launches_per_step = plan["launches"] + (1 if (comm is not None and args.collective == "nccl") else 0)
        weak = {"n_per_gpu": n, "total_bytes": world * n * 4, "ms_per_step": round(ms, 5), "value": round(value, 2),
                "unit": "GB/s", "elements_per_s": round(world * n / (ms * 1e-3), 1)}
        use_strong = args.scaling == "strong" and strong is not None
        v_ms = strong["ms_per_step"] if use_strong else ms
        v_val = strong["value"] if use_strong else value
        line = {
            "metric": METRIC, "value": round(v_val, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(v_ms, 5),
            "higher_is_better": True, "scaling": "strong" if use_strong else "weak", "vs_baseline": None,
            "dtype": "f32", "data": "synthetic", "config": workload_config(args, world, plan, comm is not None),
            "elements_per_s": strong["elements_per_s"] if use_strong else round(world * n / (ms * 1e-3), 1),
            "launch": "cuda-graph replay of the K steps" if comm is None else
                      f"stream (K sharded calls; cross-GPU combine: {args.collective})",
            "stream_launched": None if stream_ms is None else {
                "ms_per_step": round(stream_ms, 5), "value": round(world * n * 4 / (stream_ms * 1e-3) / 1e9, 2)},
            "frac_of_hbm_peak": round(v_val / world / peak, 4),
            "weak_scaling": weak, "strong_scaling": strong,
            "roofline": roofline, "e2e": e2e,
            "clocks": (strong_clocks if use_strong else clocks).summary(),
            "gpu_launches": args.steps * launches_per_step,
            "gpu": gpu_identity(local),
            "env": software_env(dev),
        }
        if use_strong:
            line["config"]["workload"] = (f"fp32 sum of one {args.strong_total}-element array split over {world} GPU(s) "
                                          f"-- BASELINE configs[4] strong scaling")
            line["config"]["total_bytes"] = args.strong_total * 4
        if comm_info is not None:
            line["comm"] = comm_info
        if decomposition is not None:
            line["sharded_decomposition"] = decomposition
        if cross_check is not None:
            line["cross_rank_check"] = cross_check
        if collective_note is not None:
            line["config"]["collective_note"] = collective_note
        if args.share_gpu:
            line["test_mode"] = "--share-gpu: all ranks on one GPU (code-path check, not a scaling number)"
        if cpu is not None:
            line["cpu_baseline"] = cpu
            line["cpu_openmp"] = cpu_omp
        line["paper_context"] = paper_context(sweep)
        if sweep is not None:
            line["sweep"] = sweep
            line["small_array_latency"] = latency
            line["batched"] = batched
            line["segmented"] = segmented
            line["ops_1GiB"] = ops_1gib
            line["histogram"] = hist
            line["config5_8GiB_one_gpu"] = big
            line["config1_int32_1M"] = cfg1
            line["config3_64M_atomic_vs_tree"] = cfg3
        if ncu_s is not None:
            line["ncu"] = {k: ncu_s[k] for k in ("source", "dram_pct_of_peak", "duration_us") if k in ncu_s}
        print(json.dumps(line), flush=True)
    if comm is not None:
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()  # no member may unmap its team buffer while others still use it
        for name in ("nvls", "team", "nccl"):  # the NVLS window before the communicator it lives on
            if combines.get(name) is not None:
                combines[name].destroy()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
