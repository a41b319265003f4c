python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
REDUCE_HIST_CLUSTER=1 timeout 300 python -m pytest tests/test_histogram_gpu.py -x -q > gpurun_out/hist_cl_tests.log 2>&1; tail -1 gpurun_out/hist_cl_tests.log
timeout 300 python tools/seg_bench.py --only histogram --tag default 2>&1 | grep 65536
REDUCE_HIST_CLUSTER=1 timeout 300 python tools/seg_bench.py --only histogram --tag cluster 2>&1 | grep 65536
