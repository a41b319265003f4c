# A/B: abtest/lib_*.so -- histogram tests + timings for all, segbal tests + timings
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rep in 1 2; do
for f in abtest/lib_*.so; do
  name=$(basename $f .so)
  cp $f $LIB
  if [ $rep = 1 ]; then
    timeout 600 python -m pytest tests/test_histogram_gpu.py -x -q > /tmp/t_$name.log 2>&1
    echo "$name hist tests: $(tail -1 /tmp/t_$name.log)"
    case $name in base|f6i5|vpl*|seg*)
      timeout 600 python -m pytest tests/test_segbal_gpu.py -x -q > /tmp/s_$name.log 2>&1
      echo "$name segbal tests: $(tail -1 /tmp/s_$name.log)";;
    esac
  fi
  timeout 300 python tools/seg_bench.py --only segmented --tag $name 2>&1 | grep '"auto"'
  timeout 300 python tools/seg_bench.py --only histogram --tag $name 2>&1 | grep '65536\|"nbins": 256,'
done
done
cp /tmp/lib_orig.so $LIB
