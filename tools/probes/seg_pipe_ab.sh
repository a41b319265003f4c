#!/usr/bin/env bash
# A/B of the segmented kernel's pipeline depth (RB_SEG_PIPE = segments whose
# first-round loads are issued together).  Run on the GPU box from the repo
# root; rebuilds the library per setting, restores the default build at the end.
set -u
mkdir -p gpurun_out
for P in ${PIPES:-1 2 4}; do
  REDUCE_B200_NVCC_FLAGS="-DRB_SEG_PIPE=$P" python -c "
import importlib.util
spec = importlib.util.spec_from_file_location('b', 'paper_conf_cgo_gonzalohghmh19_b200/_build.py')
m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m); m.build(force=True)"
  timeout 600 python tools/seg_bench.py --tag pipe$P >> gpurun_out/seg_pipe_ab.jsonl 2>> gpurun_out/seg_pipe_ab.err
done
python -c "
import importlib.util
spec = importlib.util.spec_from_file_location('b', 'paper_conf_cgo_gonzalohghmh19_b200/_build.py')
m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m); m.build(force=True)"
