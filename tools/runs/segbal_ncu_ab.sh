# per-kernel device times of the segmented workload for each abtest/lib_*.so (ncu launch list)
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
for f in abtest/lib_*.so; do
  name=$(basename $f .so)
  cp $f $LIB
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_segbal --csv \
     --log-file gpurun_out/segbal_ncu_$name.csv python tools/segbal_workload.py > /dev/null 2>&1
done
cp /tmp/lib_orig.so $LIB
