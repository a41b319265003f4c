python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^k_segbal$" --launch-skip 3 -c 1 \
  -o gpurun_out/segbal_full -f python tools/segbal_workload.py > gpurun_out/ncu_segbal.log 2>&1
ncu -i gpurun_out/segbal_full.ncu-rep --page source --csv --print-source sass > gpurun_out/segbal_source_sass.csv 2>/dev/null
ncu -i gpurun_out/segbal_full.ncu-rep --page source --csv > gpurun_out/segbal_source.csv 2>/dev/null
ncu -i gpurun_out/segbal_full.ncu-rep --page details --csv > gpurun_out/segbal_details.csv 2>/dev/null
