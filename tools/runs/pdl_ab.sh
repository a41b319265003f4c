python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
rm -f gpurun_out/pdl_ab.jsonl
for rnd in 1 2; do
for v in "default:" "nopdl:REDUCE_NO_PDL=1" "noprefetch:REDUCE_NO_PREFETCH=1" "noearly:REDUCE_NO_EARLY=1"; do
  tag=${v%%:*}; envs=${v#*:}
  env $envs timeout 300 python tools/probes/sweep_ab.py $tag >> gpurun_out/pdl_ab.jsonl 2>>gpurun_out/pdl_ab.err
done; done
