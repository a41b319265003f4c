"""BASELINE.md's Results table from one bench.py JSON line.

Usage: python tools/results_table.py profiles/r02_bench.json  (prints markdown)

Rows: the headline (configs[1] largest point), every C2 sweep point (U[0,1)),
C1 (int32 1 M, both distributions and modes), C3 (int32 / fp64 at 2^26,
atomic vs tree), C4 (small-array latency), C5 at N = 1 (2^31 fp32 on one GPU).
Columns as BASELINE.md's template: time, GB/s, elements/s, % of the nominal
8 TB/s, % of MEASURED_PEAKS hbm_gbs, ncu DRAM % (headline only), the CPU oracle
(1 core) and OpenMP rates where the bench measured them, and correctness.
"""
import json
import sys


def main():
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    peak = d["roofline"]["peak"]
    ncu = d.get("ncu", {}).get("dram_pct_of_peak")
    cpu = d.get("cpu_baseline", {}).get("value")
    omp = d.get("cpu_openmp", {}).get("value")
    rows = []

    def row(cfg, dt, n, variant, us, nbytes, ncu_pct="", cpu_gbs="", omp_gbs="", ok=""):
        gbs = nbytes / (us * 1e-6) / 1e9
        rows.append(f"| {cfg} | {dt} | {n} | {variant} | {us:.3f} | {gbs:.1f} | {n_int(n) / (us * 1e-6):.3g} | "
                    f"{100 * gbs / 8000:.1f} | {100 * gbs / peak:.1f} | {ncu_pct} | {cpu_gbs} | {omp_gbs} | {ok} |")

    def n_int(n):
        return int(str(n).split()[0])

    v = d["config"]["variant"]
    row("C2 headline (2^28)", "fp32 sum", 1 << 28, f"gc{v['grid_combine']} {v['grid']}x{v['block']} u{v['unroll']}",
        d["ms_per_step"] * 1e3, (1 << 28) * 4, f"{ncu:.1f}" if ncu else "", f"{cpu:.2f}" if cpu else "",
        f"{omp:.1f}" if omp else "", "G1+G2 (tests)")
    for e in d.get("sweep", []):
        if e["dist"] != "U[0,1)":
            continue
        c_o = e.get("cpu_oracle_us")
        c_p = e.get("cpu_omp_us")
        row(f"C2 sweep 2^{e['log2_n']}", "fp32 sum", e["n"], e["variant"], e["us"], e["n"] * 4, "",
            f"{e['n'] * 4 / (c_o * 1e-6) / 1e9:.2f}" if c_o else "", f"{e['n'] * 4 / (c_p * 1e-6) / 1e9:.1f}" if c_p else "",
            f"CUB {e['cub_us']} us ({e['speedup_vs_cub']}x)" if e.get("cub_us") else "")
    for e in d.get("config1_int32_1M") or []:
        row(f"C1 {e['dist']} {e['mode']}", "int32 sum", e["n"], e["variant"], e["gpu_us"], e["n"] * 4, "",
            f"{e['n'] * 4 / (e['cpu_oracle_us'] * 1e-6) / 1e9:.2f}", "", "bit-exact" if e["bit_exact"] else "MISMATCH")
    for r in d.get("config3_64M_atomic_vs_tree") or []:
        es = 8 if r["dtype"] == "float64" else 4
        for arm in ("atomic", "tree"):
            a = r[arm]
            extra = f", {a['distinct_results_20_runs']} distinct in 20 runs" if "distinct_results_20_runs" in a else ""
            row(f"C3 {arm}", f"{r['dtype']} {r['op']}", r["n"], f"{a['grid_combine']} {a['grid']}x{a['block']} u{a['unroll']}",
                a["us"], r["n"] * es, "", "", "", ("bit-exact (tests)" if r["op"] != "sum" or r["dtype"] == "int32"
                                                 else "G1+G2 (tests)") + extra)
    for e in d.get("small_array_latency") or []:
        row(f"C4 latency", f"{e['dtype']} sum", e["n"], "auto (graph)", e["graph_us"], e["n"] * 4, "", "", "",
            f"stream b2b {e['stream_b2b_us']} us, host wall {e['host_wall_us']} us")
    st = d.get("strong_scaling")
    if st:
        row(f"C5 N={d['n_gpus']} (strong)", "fp32 sum", st["total_elements"], st.get("launch", ""),
            st["ms_per_step"] * 1e3, st["total_bytes"], "", "", "", "sharded check" if "cross_rank_check" in st else "")
    print("| config | dtype / op | n | variant | t (µs) | GB/s | elem/s | % of 8 TB/s | % of "
          f"{peak:.0f} GB/s | ncu DRAM % | CPU oracle GB/s (1 core) | OpenMP GB/s | correctness / context |")
    print("|---|---|---|---|---|---|---|---|---|---|---|---|---|")
    print("\n".join(rows))


if __name__ == "__main__":
    main()
