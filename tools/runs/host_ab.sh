LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rnd in 1 2; do for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  echo "$name $(tools/latency_bench | head -c 600)"
  python tools/probes/py_overhead.py $name
done; done
cp /tmp/lib_orig.so $LIB
