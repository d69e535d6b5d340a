V=paper_conf_sc_markidis23_b200
bash tools/ab_run.sh "h2 l2 h3 l3 h4 q0" 1 $V/_variants/libsvb200_cplanes.so $V/libsvb200.so
timeout 900 python -m pytest tests/test_gpu_apply.py tests/test_gpu_circuit.py -m gpu -x -q 2>&1 | tail -2
