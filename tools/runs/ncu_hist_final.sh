# ncu --set full of the shipped histogram kernels: fp32 256 bins (k_histogram, shared bins)
# and fp32 65536 bins (k_histogram16r), 1 GiB each, second call of each
cat > /tmp/hw2.py <<'PY'
import sys, torch
sys.path.insert(0, '.')
import paper_conf_cgo_gonzalohghmh19_b200 as rb
x = torch.rand(1 << 28, device='cuda')
for _ in range(2):
    rb.histogram(x, 0.0, 1.0, 256)
    rb.histogram(x, 0.0, 1.0, 65536)
torch.cuda.synchronize()
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_histogram" --launch-skip 2 -c 2 \
  -o gpurun_out/hist_final -f python /tmp/hw2.py > gpurun_out/ncu_hist_final.log 2>&1
ncu -i gpurun_out/hist_final.ncu-rep --page details --csv > gpurun_out/hist_final_details.csv 2>/dev/null
ncu -i gpurun_out/hist_final.ncu-rep --page raw --csv --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed,launch__registers_per_thread,launch__grid_size,launch__block_size > gpurun_out/hist_final_raw.csv 2>/dev/null
