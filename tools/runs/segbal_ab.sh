# segbal A/B: abtest/lib_*.so -- segbal + segmented parity tests, then timings (twice)
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rep in 1 2; do
for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  if [ $rep = 1 ]; then
    timeout 600 python -m pytest tests/test_segbal_gpu.py -x -q > /tmp/s_$name.log 2>&1
    echo "$name segbal tests: $(tail -1 /tmp/s_$name.log)"
    grep -E "^FAILED|Error" /tmp/s_$name.log | head -3
  fi
  timeout 300 python tools/seg_bench.py --only segmented --tag $name 2>&1 | grep '"auto"'
done; done
cp /tmp/lib_orig.so $LIB
