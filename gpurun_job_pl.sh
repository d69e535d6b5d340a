O=gpurun_out/r4; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_fp64.py tests/test_gpu_multiproc.py -q > $O/pytest.log 2>&1; tail -15 $O/pytest.log
V=paper_conf_sc_markidis23_b200/_variants
timeout 600 python tools/ab_step.py 2 $V/libsvb200_base.so $V/libsvb200_r4.so > $O/ab30.txt 2>&1; cat $O/ab30.txt
AB_PIN=3 timeout 600 python tools/ab_step.py 1 $V/libsvb200_base.so $V/libsvb200_r4.so > $O/ab30p3.txt 2>&1; cat $O/ab30p3.txt
AB_N=32 AB_D=20 AB_PIN=3 timeout 900 python tools/ab_step.py 2 $V/libsvb200_base.so $V/libsvb200_r4.so > $O/ab32.txt 2>&1; cat $O/ab32.txt
AB_N=32 AB_D=20 timeout 900 python tools/ab_step.py 1 $V/libsvb200_base.so $V/libsvb200_r4.so > $O/ab32p4.txt 2>&1; cat $O/ab32p4.txt
