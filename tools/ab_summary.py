"""Summarise an A/B log of tools/seg_bench.py lines (tag lib_<name>): best us per case and variant.
Usage: python tools/ab_summary.py LOG"""
import collections
import json
import sys

d = collections.defaultdict(lambda: collections.defaultdict(list))
for line in open(sys.argv[1]):
    if line.startswith("{"):
        r = json.loads(line)
        k = (r["kind"], r.get("dtype", ""), r.get("nbins", f"{r.get('dist', '')}{r.get('mean_len', '')}"))
        d[k][r["tag"].removeprefix("lib_")].append(r["us"])
    elif line.strip():
        print(line.strip())
for k, v in d.items():
    print(k, {t: min(u) for t, u in v.items()})
