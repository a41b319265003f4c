python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
B="python bench.py --steps 20 --warmup 5 --no-sweep --no-cpu --no-e2e --strong-total 0"
timeout 900 ncu --graph-profiling graph --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum --csv \
  --log-file gpurun_out/ncu_graphs_nc.csv $B > gpurun_out/ncu_graphs_nc.log 2>&1
$B > gpurun_out/bench_plain.json 2>/dev/null
