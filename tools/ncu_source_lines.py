"""Aggregate an ncu source page (--page source --csv --print-source cuda,sass)
per CUDA source line: share of executed instructions and of stall samples.
Usage: python tools/ncu_source_lines.py CSV [TOP]"""
import collections
import csv
import sys

rows = csv.reader(open(sys.argv[1]))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
agg = collections.defaultdict(lambda: [0, 0, ""])
tot = [0, 0]
cur, hdr, line, src = None, None, None, ""
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None:
        continue
    if r[0] != "":
        line, src = r[0], r[1]
    try:
        ie = int(r[hdr.index("Instructions Executed")] or 0)
        s = int(r[hdr.index("# Samples")] or 0)
    except (ValueError, IndexError):
        continue
    k = (cur, line)
    agg[k][0] += ie
    agg[k][1] += s
    agg[k][2] = src.strip()[:70]
    tot[0] += ie
    tot[1] += s
print("total warp instructions", tot[0], "samples", tot[1])
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top]:
    print(f"{k[0]:22s}:{k[1]:>4s} inst {v[0] / tot[0] * 100:5.1f}% samp {v[1] / tot[1] * 100:5.1f}%  {v[2]}")
