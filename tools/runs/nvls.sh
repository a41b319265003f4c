python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_nvls_gpu.py tests/test_multi_gpu.py tests/test_team_gpu.py -x -q -rs > gpurun_out/nvls.log 2>&1; echo "rc=$?" >> gpurun_out/nvls.log
