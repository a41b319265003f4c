python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_early_loads_gpu.py -x -q > gpurun_out/parity.log 2>&1; echo "rc=$?" >> gpurun_out/parity.log
rm -f gpurun_out/packed_ab.jsonl
python tools/probes/sweep_ab.py packed >> gpurun_out/packed_ab.jsonl 2>>gpurun_out/packed_ab.err
python tools/probes/sweep_ab.py packed_regs --input-ready >> gpurun_out/packed_ab.jsonl 2>>gpurun_out/packed_ab.err
