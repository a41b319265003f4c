python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/tune.py --out gpurun_out/tune_r02b.json > gpurun_out/tune_r02b.log 2>&1
python tools/tune.py --ops sum_accurate --dtypes float32 float64 --out gpurun_out/tune_r02b_acc.json > gpurun_out/tune_r02b_acc.log 2>&1
