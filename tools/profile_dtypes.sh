#!/usr/bin/env bash
# ncu metrics SURVEY 8(d) names, for k_reduce at 2^28 int32 / fp32 and 2^26
# fp64 (sum, min, max), cold cache per launch.  GPU box, repo root.
set -u
mkdir -p gpurun_out
timeout 900 ncu --kernel-name regex:k_reduce --cache-control all --clock-control none \
  --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_read.sum.per_second,dram__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors_srcunit_tex_op_read.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,smsp__inst_executed_op_global_ld.sum,launch__grid_size,launch__block_size,launch__registers_per_thread \
  --csv --log-file gpurun_out/ncu_dtypes.csv python tools/ncu_dtypes_workload.py > gpurun_out/ncu_dtypes.log 2>&1
echo "ncu rc=$?"
