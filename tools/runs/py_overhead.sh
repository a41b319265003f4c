python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
cp paper_conf_cgo_gonzalohghmh19_b200/__init__.py /tmp/init_new.py
cp tools/runs/init_old.py paper_conf_cgo_gonzalohghmh19_b200/__init__.py
python tools/probes/py_overhead.py old
cp /tmp/init_new.py paper_conf_cgo_gonzalohghmh19_b200/__init__.py
python tools/probes/py_overhead.py new
python -m pytest tests/test_parity_gpu.py -x -q 2>&1 | tail -1
