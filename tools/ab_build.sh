#!/usr/bin/env bash
# Build one A/B variant of the library: bash tools/ab_build.sh NAME "-DFLAG=V ..."
# -> abtest/lib_NAME.so (the in-tree library keeps that variant until rebuilt)
set -eu
cd "$(dirname "$0")/.."
mkdir -p abtest
REDUCE_B200_NVCC_FLAGS="$2" python -c "import __graft_entry__ as g; g._load_build_module().build(force=True)"
cp paper_conf_cgo_gonzalohghmh19_b200/libreduce_b200.so "abtest/lib_$1.so"
