python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
export MID_AB_ONLY=auto,twopass_256x2,atomic_256x4,atomic_256x2,cub MID_AB_SIZES=19,20,21
python tools/probes/mid_ab.py lib
tools/probes/probe_twokernel
