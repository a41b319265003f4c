python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_segbal_gpu.py tests/test_segmented_gpu.py tests/test_accurate_gpu.py -x -q > gpurun_out/seg_tests.log 2>&1; echo "rc=$?" >> gpurun_out/seg_tests.log
