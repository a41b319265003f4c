# A/B of the pre-dependency L2 prefetch depth (REDUCE_PREFETCH_MB) and early register loads
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
rm -f gpurun_out/prefetch_ab.jsonl
for v in "off:REDUCE_NO_EARLY=1" "pf0:REDUCE_PREFETCH_MB=0" "pf16:REDUCE_PREFETCH_MB=16" "pf32:REDUCE_PREFETCH_MB=32" "pf64:REDUCE_PREFETCH_MB=64" "regs32:REDUCE_PREFETCH_MB=32" "regs0:REDUCE_PREFETCH_MB=0"; do
  tag=${v%%:*}; envs=${v#*:}
  extra=""; case $tag in regs*) extra="--input-ready";; esac
  env $envs timeout 300 python tools/probes/sweep_ab.py $tag $extra >> gpurun_out/prefetch_ab.jsonl 2>>gpurun_out/prefetch_ab.err
done
