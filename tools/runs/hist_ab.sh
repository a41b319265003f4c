# A/B of histogram build variants (abtest/lib_<name>.so): parity tests, then tools/seg_bench.py --only histogram
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so)
  cp $f $LIB
  timeout 300 python -m pytest tests/test_histogram_gpu.py -x -q > /tmp/t_$name.log 2>&1
  echo "$name tests: $(tail -1 /tmp/t_$name.log)"
  timeout 300 python tools/seg_bench.py --only histogram --tag $name 2>&1 | grep histogram
done
cp /tmp/lib_orig.so $LIB
