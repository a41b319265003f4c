# segbal A/B: parity tests (segbal + segmented), per-kernel split, segmented timings twice
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  timeout 600 python -m pytest tests/test_segbal_gpu.py tests/test_segmented_gpu.py -x -q > /tmp/s_$name.log 2>&1
  echo "$name seg tests: $(tail -1 /tmp/s_$name.log)"
  grep -E "^FAILED|Error" /tmp/s_$name.log | head -3
  python tools/probes/segbal_split.py | sed "s/}/, \"tag\": \"$name\"}/" | grep -v '"all"'
done
for rep in 1 2; do for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  timeout 300 python tools/seg_bench.py --only segmented --tag $name 2>&1 | grep '"auto"'
done; done
cp /tmp/lib_orig.so $LIB
