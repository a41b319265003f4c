python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
rm -f gpurun_out/big_ab.jsonl
for i in 1 2; do
for v in "noearly:REDUCE_NO_EARLY=1" "default:" "noprefetch:REDUCE_NO_PREFETCH=1" "nopdl:REDUCE_NO_PDL=1"; do
  tag=${v%%:*}; envs=${v#*:}
  env $envs python tools/probes/big_ab.py $tag >> gpurun_out/big_ab.jsonl 2>>gpurun_out/big_ab.err
done; done
