set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gputests.log
for v in "off:REDUCE_NO_EARLY=1" "prefetch:" "regs:" ; do
  tag=${v%%:*}; envs=${v#*:}
  extra=""; [ "$tag" = regs ] && extra="--input-ready"
  env $envs timeout 300 python tools/probes/sweep_ab.py $tag $extra >> gpurun_out/early_ab.jsonl 2>>gpurun_out/early_ab.err
done
