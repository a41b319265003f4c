"""Summarise a round's ncu captures into profiles/ (the numbers bench.py quotes).

  python tools/ncu_summarize.py gpurun_out/k_reduce_full_raw.csv gpurun_out/ncu_launches.csv r01

writes profiles/ncu_summary.json (dominant kernel: duration, DRAM bytes per
launch vs the algorithmic bytes, % of ncu's DRAM peak, occupancy, registers)
and profiles/<round>_ncu_launch_shares.json (per kernel name: launches, total
and mean device time, share of the profiled time) from the launch list.
"""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def scale(v, unit):
    f = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3}.get(unit, 1)
    return float(v.replace(",", "")) * f


def full_summary(raw_csv, n_bytes):
    rows = list(csv.reader(open(raw_csv)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    g = lambda k: (vals[hdr.index(k)], units[hdr.index(k)])
    rd = scale(*g("dram__bytes_read.sum"))
    wr = scale(*g("dram__bytes_write.sum"))
    dur = scale(*g("gpu__time_duration.sum"))
    return {
        "source": f"{os.path.relpath(raw_csv, ROOT)} (ncu --set full --clock-control none --import-source on, "
                  f"bench.py launch config)",
        "kernel": g("Kernel Name")[0], "grid": g("Grid Size")[0], "block": g("Block Size")[0],
        "duration_us": round(dur, 3),
        "dram_bytes_read": int(rd), "dram_bytes_write": int(wr), "dram_bytes_per_launch": int(rd + wr),
        "algorithmic_bytes_per_launch": n_bytes,
        "traffic_over_algorithmic": round((rd + wr) / n_bytes, 5),
        "dram_pct_of_peak": round(float(g("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed")[0]), 3),
        "dram_read_TBps": round(rd / dur / 1e6, 3),
        "achieved_occupancy_pct": round(float(g("sm__warps_active.avg.pct_of_peak_sustained_active")[0]), 2),
        "registers_per_thread": int(float(g("launch__registers_per_thread")[0])),
        "inst_executed": int(float(g("smsp__inst_executed.sum")[0])),
        "note": "ncu replays with caches flushed and launches serialised: its duration is one cold launch "
                "(ramp-up + drain); the bench's graph-timed steps overlap neighbours through PDL",
    }


def launch_shares(launch_csv):
    lines = [l for l in open(launch_csv) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    agg = collections.OrderedDict()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        t = scale(r["Metric Value"], r["Metric Unit"])
        key = (r["Kernel Name"], r.get("Grid Size", ""), r.get("Block Size", ""))
        a = agg.setdefault(key, {"launches": 0, "total_us": 0.0})
        a["launches"] += 1
        a["total_us"] += t
    tot = sum(a["total_us"] for a in agg.values()) or 1.0
    out = []
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["total_us"]):
        out.append({"kernel": k[0], "grid": k[1], "block": k[2], "launches": a["launches"], "total_us": round(a["total_us"], 3),
                    "mean_us": round(a["total_us"] / a["launches"], 3), "share": round(a["total_us"] / tot, 4)})
    return {"source": f"{os.path.relpath(launch_csv, ROOT)} (ncu --metrics gpu__time_duration.sum "
                      f"--clock-control none, the bench command; cold, serialised launches)",
            "kernels": out}


def main():
    raw, launches, rnd = sys.argv[1], sys.argv[2], sys.argv[3]
    n_bytes = int(sys.argv[4]) if len(sys.argv) > 4 else (1 << 28) * 4
    prof = os.path.join(ROOT, "profiles")
    s = full_summary(raw, n_bytes)
    with open(os.path.join(prof, "ncu_summary.json"), "w") as f:
        json.dump(s, f, indent=1)
    sh = launch_shares(launches)
    with open(os.path.join(prof, f"{rnd}_ncu_launch_shares.json"), "w") as f:
        json.dump(sh, f, indent=1)
    print(json.dumps(s, indent=1))
    for k in sh["kernels"][:6]:
        print(k)


if __name__ == "__main__":
    main()
