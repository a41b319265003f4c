python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 bash tests/sanitize.sh > gpurun_out/sanitize.log 2>&1; echo "sanitize rc=$?"; grep "==" gpurun_out/sanitize.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
