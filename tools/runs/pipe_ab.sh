LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rep in 1 2; do for f in abtest/lib_*.so; do name=$(basename $f .so); cp $f $LIB
  if [ $rep = 1 ]; then timeout 900 python -m pytest tests/test_parity_gpu.py -x -q > /tmp/p_$name.log 2>&1; echo "$name parity: $(tail -1 /tmp/p_$name.log)"; fi
  python tools/probes/pipe_ab.py $name; done; done
cp /tmp/lib_orig.so $LIB
