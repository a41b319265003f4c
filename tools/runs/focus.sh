python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x -k "graph or concurrent or team or bench or per_thread" > gpurun_out/focus.log 2>&1; echo "rc=$?" >> gpurun_out/focus.log
