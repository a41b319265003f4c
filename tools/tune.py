#!/usr/bin/env python
"""Autotuner -> csrc/dispatch_table.inc (step S0's table).

The paper tunes every version with every tunable at the largest size with "a
simple script" and observes that the best version changes with array
size and GPU.  This does the same on the B200, per size: every
candidate (block combine x grid combine x block x unroll x grid cap) is timed
as device time per call (CUDA graph of R calls over cold input regions, see
tools/cudatiming.py), and the fastest candidate per (dtype, op, mode, log2
bytes) becomes a table row.  Results are also written as JSON for the record.

Usage (on the GPU box):
  python tools/tune.py --dtypes float32 --ops sum --modes fast --out gpurun_out/tune.json
  python tools/tune.py --emit gpurun_out/tune.json [more.json ...]  # write dispatch_table.inc
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

ELEM = {"int32": 4, "float32": 4, "float64": 8}
DT = {"int32": 0, "float32": 1, "float64": 2}
OPC = {"sum": 0, "min": 1, "max": 2, "sum_accurate": 3}
MODE = {"fast": 0, "deterministic": 1}
MAXBLK = lambda dt, op, u: 512 if (u >= 8 or (dt == "float64" and op != "sum" and u >= 2)
                                   or (op == "sum_accurate" and u >= 4)) else 1024


def candidates(dtype, op, mode, lb):
    gcs = [1, 2, 3, 5] if mode == "fast" else [2, 3, 5]
    if op == "sum_accurate" and dtype == "float64":
        gcs = [g for g in gcs if g != 1]  # double-double: no value atomics
    out = []
    if lb <= 18:
        for blk, u in itertools.product((32, 128, 256, 512, 1024), (1, 2, 4)):
            out.append(dict(block=blk, unroll=u, grid_combine=0, block_combine=0, grid=-1))
    if lb >= 12:
        for blk, u, gc in itertools.product((128, 256, 512), (1, 2, 4, 8), gcs):
            out.append(dict(block=blk, unroll=u, grid_combine=gc, block_combine=0, grid=-1))
        for blk, u, gc in itertools.product((128, 256, 512), (4, 8, 16), gcs):
            if blk * u * 32 <= 128 * 1024:
                out.append(dict(block=blk, unroll=u, grid_combine=gc, block_combine=0, grid=-1, stage=2))
        for bc in (1, 2, 3):
            if (mode == "deterministic" or (op == "sum_accurate" and dtype == "float64")) and bc in (1, 2):
                continue
            out.append(dict(block=256, unroll=2, grid_combine=gcs[0], block_combine=bc, grid=-1))
    if 10 <= lb <= 26:
        for blk, u, c in itertools.product((256, 512, 1024), (1, 2, 4), (4, 8, 16)):
            out.append(dict(block=blk, unroll=u, grid_combine=4, block_combine=0, grid=c))
        for blk, u, c in itertools.product((256, 512), (8, 16), (8, 16)):
            if blk * u * 32 <= 128 * 1024:
                out.append(dict(block=blk, unroll=u, grid_combine=4, block_combine=0, grid=c, stage=2))
    if lb >= 24:
        for blk, g, gc in itertools.product((256, 512), (148 * 2, 148 * 4, 148 * 8), (gcs[0], 5)):
            out.append(dict(block=blk, unroll=4, grid_combine=gc, block_combine=0, grid=g))
    for c in out:
        c.setdefault("stage", 1)
    ok = lambda c: (c["block"] <= (512 if op == "sum_accurate" else 1024) if c["stage"] == 2
                    else c["block"] <= MAXBLK(dtype, op, c["unroll"]))
    return [c for c in out if ok(c)]


def run(args):
    import torch
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    from cudatiming import time_calls, disjoint_regions

    dev = torch.device("cuda", 0)
    stream = torch.cuda.Stream(dev)
    pool_bytes = 2 << 30
    pools = {}
    results = []
    t_start = time.time()
    for dtype in args.dtypes:
        tdt = getattr(torch, dtype)
        if dtype not in pools:
            p = torch.empty(pool_bytes // ELEM[dtype], dtype=tdt, device=dev)
            if dtype == "int32":
                p.random_(-1000, 1000)
            else:
                p.uniform_(-1, 1)
            pools[dtype] = p
        pool = pools[dtype]
        rb.prepare(stream, pool.numel())
        out = torch.empty(4096, dtype=tdt, device=dev)
        for op, mode in itertools.product(args.ops, args.modes):
            for lb in range(args.min_lb, args.max_lb + 1):
                nbytes = 1 << lb
                n = nbytes // ELEM[dtype]
                # >= 20 calls per timed graph; regions repeat only when each is > 2x L2
                R = max(20, min(100, (400 << 20) // nbytes))
                warm, timed = disjoint_regions(pool, R, n)
                # every candidate timed in `rounds` interleaved rounds (box-level
                # drift hits all candidates alike), the median per candidate decides
                cands = candidates(dtype, op, mode, lb)
                times = [[] for _ in cands]
                failed = set()
                for rnd in range(args.rounds):
                    for ci, c in enumerate(cands):
                        if ci in failed:
                            continue
                        opts = rb.make_opts(mode=mode, input_ready=args.input_ready, **c)
                        k = [0]

                        def launch(t, opts=opts):
                            i = k[0] = (k[0] + 1) % 4096
                            rb.reduce_ptr(DT[dtype], op, t.data_ptr(), t.numel(), out[i:i + 1].data_ptr(),
                                          stream.cuda_stream, opts)
                        try:
                            times[ci].append(time_calls(launch, warm, timed, stream, repeats=1))
                        except Exception as e:  # an invalid combination: record and skip
                            results.append(dict(dtype=dtype, op=op, mode=mode, lb=lb, cfg=c, error=str(e)[:200],
                                                ready=int(args.input_ready)))
                            torch.cuda.synchronize()
                            failed.add(ci)
                best = None
                for ci, c in enumerate(cands):
                    if ci in failed or not times[ci]:
                        continue
                    s = sorted(times[ci])[len(times[ci]) // 2]
                    results.append(dict(dtype=dtype, op=op, mode=mode, lb=lb, cfg=c, us=s * 1e6,
                                        gbps=nbytes / s / 1e9, rounds_us=[round(t * 1e6, 3) for t in times[ci]],
                                        ready=int(args.input_ready)))
                    if best is None or s < best[0]:
                        best = (s, c)
                print(f"[{time.time() - t_start:7.1f}s] {dtype} {op} {mode}{' ready' if args.input_ready else ''} 2^{lb}B: best {best[0] * 1e6:8.2f} us "
                      f"{nbytes / best[0] / 1e9:8.1f} GB/s {best[1]}", flush=True)
                with open(args.out, "w") as f:
                    json.dump(results, f)
    return results


def table_rows(by, tol):
    """Pick, per (dtype, op, mode, log2 bytes), the fastest candidate -- but among
    candidates within `tol` of the fastest (timer noise) keep the previous size
    bucket's choice when it qualifies, so the table only changes where the
    measurements say it must."""
    sig = lambda c: (c["block"], c["unroll"], c["grid_combine"], c["block_combine"], c["grid"], c.get("stage", 1))
    rows = []
    groups = sorted(set(k[:3] for k in by))
    for dtype, op, mode in groups:
        lbs = sorted(k[3] for k in by if k[:3] == (dtype, op, mode))
        chosen = []
        prev = None
        for lb in lbs:
            cands = by[(dtype, op, mode, lb)]
            fastest = min(r["us"] for r in cands)
            ok = [r for r in cands if r["us"] <= fastest * (1 + tol)]
            keep = [r for r in ok if prev is not None and sig(r["cfg"]) == prev]
            pick = keep[0] if keep else min(ok, key=lambda r: r["us"])
            prev = sig(pick["cfg"])
            chosen.append((lb, pick))
        for i, (lb, pick) in enumerate(chosen):
            last = i == len(chosen) - 1
            if last or sig(chosen[i + 1][1]["cfg"]) != sig(pick["cfg"]):
                c = dict(pick["cfg"])
                c["grid"] = max(0, c["grid"])  # table: 0 = one block per tile
                rows.append((DT[dtype], OPC[op], MODE[mode], 63 if last else lb) + sig(c) +
                            (round(pick["gbps"], 1),))
        # min mirrors max when only max was tuned
        if op == "max" and (dtype, "min", mode) not in groups:
            for r in [r for r in rows if r[:3] == (DT[dtype], OPC["max"], MODE[mode])]:
                rows.append((r[0], OPC["min"]) + r[2:])
    return rows


def emit(paths, dst, tol=0.01):
    """Write dispatch_table.inc: kDispatch from the default-path measurements and
    kDispatchReady from the REDUCE_FLAG_INPUT_READY ones (tune.py --input-ready)."""
    by = {0: {}, 1: {}}
    for p in paths:  # a later file replaces earlier measurements of the same bucket
        cur = {0: {}, 1: {}}
        for r in json.load(open(p)):
            if "us" in r:
                cur[r.get("ready", 0)].setdefault((r["dtype"], r["op"], r["mode"], r["lb"]), []).append(r)
        for k in (0, 1):
            by[k].update(cur[k])
    lines = [
        "// dispatch_table.inc -- variant / launch choice per (dtype, op, mode, size).",
        "// Step S0 of DESIGN.md: the paper picks a code version per size and",
        "// architecture by tuning (P:L483); the winners change with size",
        "// (P:L681-L687, P:L691-L735, P:L739-L781).  GENERATED by tools/tune.py from",
        "// B200 measurements (device time per call, cold inputs); first match wins.",
        "// kDispatch: the default (safe) stream ordering; kDispatchReady: calls with",
        "// REDUCE_FLAG_INPUT_READY, whose first tile may be loaded before the",
        "// programmatic dependency resolves (so other launch shapes win).",
        "//",
        "// fields: dtype, op, mode, max_log2_bytes, block, unroll, grid_combine, block_combine, grid_cap, stage",
        "//   (grid_cap 0 = one block per tile; stage 1 = registers, 2 = shared memory via cp.async)",
        "//   trailing comment: measured GB/s at the bucket that ended the row",
    ]
    total = 0
    for k, name in ((0, "kDispatch"), (1, "kDispatchReady")):
        rows = table_rows(by[k], tol)
        total += len(rows)
        lines.append(f"static const DispatchEntry {name}[] = {{")
        for r in rows:
            lines.append("    {%d, %d, %d, %d, %d, %d, %d, %d, %d, %d},  // %.1f GB/s" % r)
        lines += ["    {-1, -1, -1, 63, 256, 4, -1, 0, 0, 1},  // fallback", "};"]
    lines += [f"static constexpr bool kHaveReadyTable = {'true' if by[1] else 'false'};", ""]
    open(dst, "w").write("\n".join(lines))
    print(f"wrote {total} rows to {dst}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dtypes", nargs="+", default=["int32", "float32", "float64"])
    ap.add_argument("--ops", nargs="+", default=["sum", "max"])
    ap.add_argument("--modes", nargs="+", default=["fast", "deterministic"])
    ap.add_argument("--min-lb", type=int, default=7)
    ap.add_argument("--max-lb", type=int, default=30)
    ap.add_argument("--out", default="gpurun_out/tune.json")
    ap.add_argument("--rounds", type=int, default=3, help="interleaved timing rounds per candidate (median wins)")
    ap.add_argument("--emit", nargs="*")
    ap.add_argument("--input-ready", action="store_true",
                    help="time every candidate with REDUCE_FLAG_INPUT_READY (rows for kDispatchReady)")
    ap.add_argument("--dst", default=os.path.join(ROOT, "paper_conf_cgo_gonzalohghmh19_b200", "csrc",
                                                  "dispatch_table.inc"))
    args = ap.parse_args()
    if args.emit:
        return emit(args.emit, args.dst)
    run(args)


if __name__ == "__main__":
    main()
