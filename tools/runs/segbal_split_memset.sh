python tools/probes/segbal_split.py > gpurun_out/segbal_split.txt 2>&1
LIB=paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so
cp $LIB /tmp/lib_orig.so
python tools/seg_bench.py --only histogram --tag base > gpurun_out/hist_memset.txt 2>&1
cp abtest2/lib_nomemset.so $LIB
python tools/seg_bench.py --only histogram --tag nomemset >> gpurun_out/hist_memset.txt 2>&1
cp /tmp/lib_orig.so $LIB
python tools/seg_bench.py --only histogram --tag base >> gpurun_out/hist_memset.txt 2>&1
