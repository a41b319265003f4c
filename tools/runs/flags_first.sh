# GC_FLAGS first GPU pass: build, its tests + the variant parity tests, then
# the tuner on fp32 sums (fast + deterministic) to see where FLAGS wins
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_flags_gpu.py tests/test_parity_gpu.py tests/test_accurate_gpu.py tests/test_early_loads_gpu.py -q -x > gpurun_out/flags_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/flags_tests.log
tail -3 gpurun_out/flags_tests.log
timeout 1500 python tools/tune.py --dtypes float32 --ops sum --modes fast deterministic --min-lb 14 --max-lb 30 --rounds 3 --out gpurun_out/tune_flags_f32.json > gpurun_out/tune_flags_f32.log 2>&1
tail -40 gpurun_out/tune_flags_f32.log
