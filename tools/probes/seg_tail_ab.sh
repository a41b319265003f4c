#!/usr/bin/env bash
# A/B of the segmented kernel's fold tail (RB_SEG_TAIL=1: one predicated round
# of up to U-1 loads; 0: one load at a time).  GPU box, repo root; restores the
# default build at the end.
set -u
mkdir -p gpurun_out
build() {
  REDUCE_B200_NVCC_FLAGS="$1" python -c "
import importlib.util
spec = importlib.util.spec_from_file_location('b', 'paper_conf_cgo_gonzalohghmh19_b200/_build.py')
m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m); m.build(force=True)"
}
for T in 0 1; do
  build "-DRB_SEG_TAIL=$T"
  timeout 600 python tools/seg_bench.py --tag tail$T >> gpurun_out/seg_tail_ab.jsonl 2>> gpurun_out/seg_tail_ab.err
done
build ""
