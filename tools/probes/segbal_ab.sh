#!/usr/bin/env bash
# A/B of k_segbal build variants (abtest/lib_<name>.so built locally with
# REDUCE_B200_NVCC_FLAGS): each variant is swapped in as the library, checked
# on the power-law parity cases, then timed with tools/seg_bench.py.
set -u
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so)
  cp $f $LIB
  timeout 300 python -m pytest tests/test_segbal_gpu.py -x -q -k "powerlaw or regimes" > /tmp/t_$name.log 2>&1
  echo "$name tests: $(tail -1 /tmp/t_$name.log)"
  timeout 300 python tools/seg_bench.py --only segmented --tag $name 2>&1 | grep '"auto"'
done
cp /tmp/lib_orig.so $LIB
