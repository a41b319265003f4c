# ncu --set full of the pair-counting histogram (fp32, 256 bins, 1 GiB) and of k_histogram16r (65536 bins)
cat > /tmp/hw.py <<'PY'
import sys, torch
sys.path.insert(0, '.')
import paper_conf_cgo_gonzalohghmh19_b200 as rb
x = torch.rand(1 << 28, device='cuda')
for _ in range(2):
    rb.histogram(x, 0.0, 1.0, 256)
    rb.histogram(x, 0.0, 1.0, 65536)
torch.cuda.synchronize()
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_histogram16" --launch-skip 2 -c 2 \
  -o gpurun_out/hist_pairs -f python /tmp/hw.py > gpurun_out/ncu_hist_pairs.log 2>&1
ncu -i gpurun_out/hist_pairs.ncu-rep --page details --csv > gpurun_out/hist_pairs_details.csv 2>/dev/null
ncu -i gpurun_out/hist_pairs.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/hist_pairs_source.csv 2>/dev/null
