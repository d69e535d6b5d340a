python -c "import __graft_entry__ as g; g.build()" > /dev/null
V=paper_conf_sc_markidis23_b200
SVB200_TC=i8 timeout 600 python tools/circuit_drift.py 24 14 4 5 6
timeout 600 python tools/circuit_drift.py 24 14 4 5 6
SVB200_TC=i8 timeout 600 python tools/tc_check.py
timeout 900 python -m pytest tests/test_gpu_apply.py tests/test_gpu_tc.py -m gpu -x -q 2>&1 | tail -2
SVB200_TC=i8 bash tools/ab_run.sh "h4 h5 h6" 1 $V/_variants/libsvb200_nacc4.so $V/libsvb200.so
