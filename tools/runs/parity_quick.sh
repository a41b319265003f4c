python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_early_loads_gpu.py tests/test_parity_gpu.py -x -q -rs > gpurun_out/parity.log 2>&1; echo "rc=$?" >> gpurun_out/parity.log
