# A/B: abtest/lib_*.so -- segbal parity tests + segmented timings, histogram timings
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rep in 1 2; do
for f in abtest/lib_*.so; do
  name=$(basename $f .so)
  cp $f $LIB
  if [ $rep = 1 ]; then
    timeout 600 python -m pytest tests/test_segbal_gpu.py tests/test_segmented_gpu.py -x -q > /tmp/t_$name.log 2>&1
    echo "$name seg tests: $(tail -1 /tmp/t_$name.log)"
    grep -E "FAILED|Error|assert" /tmp/t_$name.log | head -5
  fi
  timeout 300 python tools/seg_bench.py --only segmented --tag $name 2>&1 | grep '"auto"'
  timeout 300 python tools/seg_bench.py --only histogram --tag $name 2>&1 | grep '65536\|"nbins": 256,'
done
done
cp /tmp/lib_orig.so $LIB
