# ncu of the shipped segbal chunk kernel (power-law workload, second call): metric set + source view
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_segbal$" --launch-skip 3 -c 1 \
  -o gpurun_out/segbal_final -f python tools/segbal_workload.py > gpurun_out/ncu_segbal_final.log 2>&1
ncu -i gpurun_out/segbal_final.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,launch__block_size,smsp__inst_executed.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed > gpurun_out/segbal_final_raw.csv 2>/dev/null
ncu -i gpurun_out/segbal_final.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/segbal_final_source.csv 2>/dev/null
python tools/probes/segbal_split.py > gpurun_out/segbal_split_final.txt 2>&1
