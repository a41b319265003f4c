#!/usr/bin/env bash
# (The split path was reverted after this A/B -- see profiles/r01_tail_split_ab.json;
#  the script is kept as the record of how the numbers were taken.)
# A/B of the drain split of k_reduce's last tiles: (a) kernels built without
# the split path, (b) built with it but disabled (REDUCE_TAIL_SPLIT=0), (c) on.
# Default bench line + ops table each.  GPU box, repo root; restores the build.
set -u
mkdir -p gpurun_out
build() {
  REDUCE_B200_NVCC_FLAGS="$1" python -c "
import importlib.util
spec = importlib.util.spec_from_file_location('b', 'paper_conf_cgo_gonzalohghmh19_b200/_build.py')
m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m); m.build(force=True)"
}
build "-DRB_TAIL_SPLIT=0"
for i in 1 2; do python bench.py --no-cpu --no-e2e > gpurun_out/tsplit_nocode_$i.json 2>/dev/null; done
build ""
for i in 1 2; do
  REDUCE_TAIL_SPLIT=0 python bench.py --no-cpu --no-e2e > gpurun_out/tsplit_off_$i.json 2>/dev/null
  python bench.py --no-cpu --no-e2e > gpurun_out/tsplit_on_$i.json 2>/dev/null
done
