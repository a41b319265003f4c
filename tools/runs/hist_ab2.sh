# histogram A/B: abtest/lib_*.so (names ending in _nopdl run with REDUCE_NO_PDL=1) -- tests, then timings twice
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  case $name in *_nopdl) export REDUCE_NO_PDL=1;; *nopairs) export REDUCE_HIST_PAIRS=0;; *) unset REDUCE_NO_PDL REDUCE_HIST_PAIRS;; esac
  timeout 600 python -m pytest tests/test_histogram_gpu.py -x -q > /tmp/h_$name.log 2>&1
  echo "$name hist tests: $(tail -1 /tmp/h_$name.log)"
  grep -E "^FAILED|Error" /tmp/h_$name.log | head -3
done
for rep in 1 2; do for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  case $name in *_nopdl) export REDUCE_NO_PDL=1;; *nopairs) export REDUCE_HIST_PAIRS=0;; *) unset REDUCE_NO_PDL REDUCE_HIST_PAIRS;; esac
  timeout 300 python tools/seg_bench.py --only histogram --tag $name 2>&1 | grep histogram
done; done
unset REDUCE_NO_PDL
cp /tmp/lib_orig.so $LIB
