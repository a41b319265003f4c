# For each abtest/lib_<name>.so: parity subset, then large-size and sweep timings (2 interleaved rounds)
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so); cp $f $LIB
  timeout 600 python -m pytest tests/test_parity_gpu.py -x -q > /tmp/t_$name.log 2>&1
  echo "$name parity: $(tail -1 /tmp/t_$name.log)"
done
for rnd in 1 2; do
  for f in abtest/lib_*.so; do
    name=$(basename $f .so); cp $f $LIB
    timeout 300 python tools/probes/big_ab.py $name
    timeout 300 python tools/probes/sweep_ab.py $name
  done
done
cp /tmp/lib_orig.so $LIB
