LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for rep in 1 2; do for f in abtest/lib_*.so; do name=$(basename $f .so); cp $f $LIB
  python tools/probes/segbal_split.py | grep -E '"fix"|"all"' | sed "s/}/, \"tag\": \"$name\"}/"; done; done
cp /tmp/lib_orig.so $LIB
