# ncu --set full of the segbal scan and fix kernels (power-law workload, second call)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_segbal_scan|k_segbal_fix" --launch-skip 6 -c 2 \
  -o gpurun_out/segbal_aux -f python tools/segbal_workload.py > gpurun_out/ncu_segbal_aux.log 2>&1
ncu -i gpurun_out/segbal_aux.ncu-rep --page details --csv > gpurun_out/segbal_aux_details.csv 2>/dev/null
ncu -i gpurun_out/segbal_aux.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/segbal_aux_source.csv 2>/dev/null
