# Round-2 profile record (GPU box, repo root, one GPU).  Never report a number
# printed under ncu as a bench value.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
B="python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu --no-e2e --strong-total 0"
# 1. launch list of the bench command (per-launch device time, cold, serialised)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/ncu_launches.csv $B > gpurun_out/ncu_launches.log 2>&1
# 2. the graph-replayed K-step loop profiled as whole graphs: device time per graph
timeout 900 ncu --graph-profiling graph --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/ncu_graphs.csv $B > gpurun_out/ncu_graphs.log 2>&1
# 3. one full capture of the dominant kernel at the bench's launch configuration
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_reduce --launch-skip 8 -c 1 \
  -o gpurun_out/k_reduce_full -f $B > gpurun_out/ncu_full.log 2>&1
ncu -i gpurun_out/k_reduce_full.ncu-rep --page raw --csv > gpurun_out/k_reduce_full_raw.csv 2>/dev/null
ncu -i gpurun_out/k_reduce_full.ncu-rep --page details --csv > gpurun_out/k_reduce_full_details.csv 2>/dev/null
# 4. the SURVEY 8(d) metric set per dtype / op at the shipped table's shapes
bash tools/profile_dtypes.sh > gpurun_out/profile_dtypes.log 2>&1
echo done
