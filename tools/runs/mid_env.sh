python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
export MID_AB_ONLY=auto,twopass_256x2,atomic_256x4,cub MID_AB_SIZES=19,20
for v in "default:" "nopdl:REDUCE_NO_PDL=1" "noprefetch:REDUCE_NO_PREFETCH=1" "noearly:REDUCE_NO_EARLY=1"; do
  tag=${v%%:*}; envs=${v#*:}
  env $envs python tools/probes/mid_ab.py $tag
done
