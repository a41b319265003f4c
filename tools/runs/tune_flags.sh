# full re-tune with the GC_FLAGS candidates (same invocation as tune.sh)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/tune.py --out gpurun_out/tune_r02c.json > gpurun_out/tune_r02c.log 2>&1
python tools/tune.py --ops sum_accurate --dtypes float32 float64 --out gpurun_out/tune_r02c_acc.json > gpurun_out/tune_r02c_acc.log 2>&1
tail -5 gpurun_out/tune_r02c.log
