# A/B old vs new library: segbal (coalesced scan) and histogram (64-bit pair merge)
bash tools/probes/segbal_ab.sh > gpurun_out/segbal_ab2.txt 2>&1
bash tools/runs/hist_ab.sh > gpurun_out/hist_ab2.txt 2>&1
bash tools/probes/segbal_ab.sh >> gpurun_out/segbal_ab2.txt 2>&1
bash tools/runs/hist_ab.sh >> gpurun_out/hist_ab2.txt 2>&1
cat gpurun_out/segbal_ab2.txt gpurun_out/hist_ab2.txt
