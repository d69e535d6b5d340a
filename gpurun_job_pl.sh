O=gpurun_out/bm5; mkdir -p $O
V=paper_conf_sc_markidis23_b200/_variants
timeout 600 python tools/ab_step.py 3 $V/libsvb200_cur.so $V/libsvb200_bm5.so > $O/ab30.txt 2>&1; cat $O/ab30.txt
AB_N=32 AB_D=20 timeout 900 python tools/ab_step.py 1 $V/libsvb200_cur.so $V/libsvb200_bm5.so > $O/ab32.txt 2>&1; cat $O/ab32.txt
