# segmented timings only (3 repetitions), per abtest/lib_*.so
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rep in 1 2 3; do for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  timeout 300 python tools/seg_bench.py --only segmented --tag $name 2>&1 | grep '"auto"'
done; done
cp /tmp/lib_orig.so $LIB
