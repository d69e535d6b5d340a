O=gpurun_out/anyd; mkdir -p $O
V=paper_conf_sc_markidis23_b200/_variants
timeout 600 python tools/ab_step.py 3 $V/libsvb200_cur.so $V/libsvb200_anyd.so > $O/ab30.txt 2>&1; cat $O/ab30.txt
AB_N=32 AB_D=20 timeout 900 python tools/ab_step.py 2 $V/libsvb200_cur.so $V/libsvb200_anyd.so > $O/ab32.txt 2>&1; cat $O/ab32.txt
AB_PIN=3 timeout 600 python tools/ab_step.py 1 $V/libsvb200_cur.so $V/libsvb200_anyd.so > $O/ab30p3.txt 2>&1; cat $O/ab30p3.txt
SVB200_LIB=$PWD/$V/libsvb200_anyd.so timeout 900 python -m pytest tests/test_gpu_jit.py -q -k "oracle or spec or tile14 or bins" > $O/pytest.log 2>&1; tail -3 $O/pytest.log
