V=paper_conf_sc_markidis23_b200
bash tools/ab_run.sh "h1 l1 h2 l2 h3 l3 h4 l4 q0" 2 $V/_variants/libsvb200_old.so $V/libsvb200.so
SVB200_TC=i8 bash tools/ab_run.sh "h4 q0 h5 h6" 2 $V/_variants/libsvb200_old.so $V/libsvb200.so
