O=gpurun_out/remap; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py tests/test_gpu_fullsize.py tests/test_gpu_fp64.py -x -q > $O/pytest.log 2>&1; tail -3 $O/pytest.log
B=paper_conf_sc_markidis23_b200/libsvb200.so; V=paper_conf_sc_markidis23_b200/_variants/libsvb200_base.so
timeout 600 python tools/ab_step.py 3 $V $B > $O/ab30.txt 2>&1; cat $O/ab30.txt
AB_N=32 AB_D=20 timeout 900 python tools/ab_step.py 2 $V $B > $O/ab32.txt 2>&1; cat $O/ab32.txt
AB_PIN=3 timeout 600 python tools/ab_step.py 2 $V $B > $O/ab30p3.txt 2>&1; cat $O/ab30p3.txt
