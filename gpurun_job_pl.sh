O=gpurun_out/l2pf; mkdir -p $O
V=paper_conf_sc_markidis23_b200/_variants
timeout 900 python tools/ab_step.py 3 $V/libsvb200_base.so $V/libsvb200_l2pf1.so $V/libsvb200_l2pf2.so > $O/ab30.txt 2>&1; cat $O/ab30.txt
AB_PIN=5 timeout 600 python tools/ab_step.py 2 $V/libsvb200_base.so $V/libsvb200_l2pf2.so > $O/ab30_pin5.txt 2>&1; cat $O/ab30_pin5.txt
AB_N=32 AB_D=20 timeout 900 python tools/ab_step.py 2 $V/libsvb200_base.so $V/libsvb200_l2pf2.so > $O/ab32.txt 2>&1; cat $O/ab32.txt
