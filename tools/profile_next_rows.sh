#!/usr/bin/env bash
# ncu per-kernel metrics of the next-row workloads (N1 segmented / batched, N4
# histogram), second pass of tools/next_rows_workload.py.  GPU box, repo root.
set -u
mkdir -p gpurun_out
timeout 900 ncu --clock-control none --cache-control all \
  --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,launch__block_size \
  --csv --log-file gpurun_out/ncu_next_rows.csv python tools/next_rows_workload.py > gpurun_out/ncu_next_rows.log 2>&1
echo "ncu rc=$?"
