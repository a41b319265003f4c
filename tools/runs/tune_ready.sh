# tune the REDUCE_FLAG_INPUT_READY table (kDispatchReady)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/tune.py --input-ready --out gpurun_out/tune_r02c_ready.json > gpurun_out/tune_r02c_ready.log 2>&1
python tools/tune.py --input-ready --ops sum_accurate --dtypes float32 float64 --out gpurun_out/tune_r02c_ready_acc.json > gpurun_out/tune_r02c_ready_acc.log 2>&1
grep -E "float32 sum (fast|deterministic) ready 2\^(2[0-8])B" gpurun_out/tune_r02c_ready.log | cut -c1-160
