#!/usr/bin/env bash
# Registers / spills of the kernels matching a regex in one translation unit:
# bash tools/ptxas_check.sh reduce_f32.cu 'k_histogram16r'
cd "$(dirname "$0")/../paper_conf_cgo_gonzalohghmh19_b200/csrc"
NCCLI=$(python -c "import site,os;print([os.path.join(p,'nvidia/nccl/include') for p in site.getsitepackages() if os.path.exists(os.path.join(p,'nvidia/nccl/include'))][0])")
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC -I ../../include -I . -I "$NCCLI" $3 \
  -Xptxas -v -c "$1" -o /tmp/ptxas_check.o 2>&1 | grep -A3 "Compiling entry function '[^']*$2" | grep -E "Compiling|registers|spill"
