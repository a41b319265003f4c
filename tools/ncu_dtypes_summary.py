"""profiles/<round>_ncu_dtypes.json from tools/profile_dtypes.sh's CSV.

  python tools/ncu_dtypes_summary.py gpurun_out/ncu_dtypes.csv profiles/r02_ncu_dtypes.json

The workload (tools/ncu_dtypes_workload.py) launches every (dtype, op) twice;
the second launch of each pair is kept (the first pays one-time costs)."""
import csv
import json
import sys

CASES = [(dt, op) for dt in ("int32", "float32", "float64") for op in ("sum", "min", "max")]


def main():
    rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
    hdr = rows[0]
    col = {k: hdr.index(k) for k in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value")}
    by_id = {}
    for r in rows[1:]:
        i = int(r[col["ID"]])
        d = by_id.setdefault(i, {"kernel": r[col["Kernel Name"]]})
        d[r[col["Metric Name"]]] = f"{r[col['Metric Value']]} {r[col['Metric Unit']]}".strip()
    ids = sorted(by_id)
    out = []
    for k, (dt, op) in enumerate(CASES):
        if 2 * k + 1 < len(ids):
            out.append(dict(dtype=dt, op=op, **by_id[ids[2 * k + 1]]))
    json.dump({"source": "tools/profile_dtypes.sh (ncu --cache-control all --clock-control none, second launch of "
                         "each), " + (sys.argv[3] if len(sys.argv) > 3 else "current build and dispatch table"),
               "launches": out}, open(sys.argv[2], "w"), indent=1)


if __name__ == "__main__":
    main()
