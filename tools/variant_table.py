"""The paper's variant study recast on B200: from the autotuner's measurements
(profiles/tune/r01_tune_v7_early.json, graph-timed, cold inputs) print, per size,
the best time of each block combine (the paper's cooperative codelets:
Vs = shuffle/redux + shared partials, Listing 4; VA2+S = a shared atomic per
warp, Fig. 3(b); VA1 = a shared atomic per thread, Fig. 3(a); V = shared tree,
Fig. 1(c)) at the same launch shape, and of each grid combine (DIRECT = one
block, ATOMIC = "DT,A" Listing 2, TWO_PASS = second launch, LAST_BLOCK,
CLUSTER = DSMEM), each at its best launch shape -- the B200 counterpart of the
paper's per-architecture variant rankings (Fig. 6).
Usage: python tools/variant_table.py > profiles/r01_paper_variants_b200.md
"""
import collections
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BC = {0: "Vs", 1: "VA2+S", 2: "VA1", 3: "V"}
GC = {0: "DIRECT", 1: "ATOMIC", 2: "TWO_PASS", 3: "LAST_BLOCK", 4: "CLUSTER"}


def main():
    d = json.load(open(os.path.join(ROOT, "profiles", "tune", "r01_tune_v7_early.json")))
    print("# The paper's reduction variants on B200 (graph-timed µs per call, cold input)\n")
    print("Source: `profiles/tune/r01_tune_v7_early.json` (tools/tune.py), table by `tools/variant_table.py`.")
    print("Block combines are compared at the launch shape the tuner measured them at "
          "(256 threads, 2 vectors per thread, the tuner's grid combine for that size); "
          "grid combines at their best launch shape.  Bold = fastest in the row.\n")
    for dtype, op in (("int32", "sum"), ("float32", "sum"), ("float32", "max"), ("float64", "sum")):
        rows = [e for e in d if e["dtype"] == dtype and e["op"] == op and e["mode"] == "fast"]
        bc_best = collections.defaultdict(dict)
        gc_best = collections.defaultdict(dict)
        for e in rows:
            c, lb, us = e["cfg"], e["lb"], e["us"]
            if c["block"] == 256 and c["unroll"] == 2 and c.get("stage", 1) == 1 and c["grid"] == -1:
                k = (lb, c["grid_combine"])
                bc_best[k][c["block_combine"]] = min(us, bc_best[k].get(c["block_combine"], 1e9))
            if c["block_combine"] == 0:
                gc_best[lb][c["grid_combine"]] = min(us, gc_best[lb].get(c["grid_combine"], 1e9))
        print(f"## {dtype} {op}\n")
        print("| bytes | " + " | ".join(BC[b] for b in range(4)) + " | " + " | ".join(GC[g] for g in range(5)) + " |")
        print("|---|" + "---|" * 9)
        for lb in sorted(gc_best):
            # the block-combine comparison at the grid combine all four were measured with
            cand = [k for k in bc_best if k[0] == lb and len(bc_best[k]) == 4]
            bcs = bc_best[cand[0]] if cand else {}
            bmin = min(bcs.values()) if bcs else None
            gmin = min(gc_best[lb].values())
            fmt = lambda v, m: "–" if v is None else (f"**{v:.2f}**" if abs(v - m) < 1e-9 else f"{v:.2f}")
            cells = [fmt(bcs.get(b), bmin) for b in range(4)] + [fmt(gc_best[lb].get(g), gmin) for g in range(5)]
            print(f"| 2^{lb} | " + " | ".join(cells) + " |")
        print()


if __name__ == "__main__":
    main()
