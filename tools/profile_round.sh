#!/usr/bin/env bash
# Round profile recipe (run on the GPU box from the repo root, one GPU):
#   1. the default bench line            -> gpurun_out/bench.json
#   2. ncu launch list of the same command (per-launch device times, cold and
#      serialised)                       -> gpurun_out/ncu_launches.csv
#   3. one ncu --set full capture of the dominant kernel (k_reduce, the
#      bench's launch configuration)     -> gpurun_out/k_reduce_full.ncu-rep + csv
# Never report a number printed under ncu as a bench value.
set -u
mkdir -p gpurun_out
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/ncu_launches.csv python bench.py --steps 3 --warmup 3 --no-sweep --no-cpu \
  > gpurun_out/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_reduce --launch-skip 8 -c 1 \
  -o gpurun_out/k_reduce_full -f python bench.py --steps 3 --warmup 3 --no-sweep --no-cpu --no-e2e \
  > gpurun_out/ncu_full.log 2>&1
ncu -i gpurun_out/k_reduce_full.ncu-rep --page details --csv > gpurun_out/k_reduce_full_details.csv 2>/dev/null
ncu -i gpurun_out/k_reduce_full.ncu-rep --page raw --csv > gpurun_out/k_reduce_full_raw.csv 2>/dev/null
tail -1 gpurun_out/bench.json | head -c 400; echo
