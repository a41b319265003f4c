python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_bench_gpu.py -x -q > gpurun_out/bench_tests.log 2>&1; echo "rc=$?" >> gpurun_out/bench_tests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench_tests.log
