#!/usr/bin/env bash
# Swap each abtest/lib_<name>.so in as the library and run a probe script with
# the name as its tag: bash tools/probes/lib_ab.sh tools/probes/sweep_ab.py
set -u
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so)
  cp $f $LIB
  timeout 600 python "$1" "$name"
done
cp /tmp/lib_orig.so $LIB
