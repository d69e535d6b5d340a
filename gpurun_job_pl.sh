O=gpurun_out/tie; mkdir -p $O
B=paper_conf_sc_markidis23_b200/libsvb200.so
for r in 1 2 3; do for b in 1 5; do AB_BEAM=$b timeout 600 python tools/ab_step.py 1 $B | sed "s/^/beam$b /"; done; done > $O/ab30.txt 2>&1; cat $O/ab30.txt
for r in 1 2; do for b in 1 5; do AB_N=32 AB_D=20 AB_BEAM=$b timeout 600 python tools/ab_step.py 1 $B | sed "s/^/beam$b /"; done; done > $O/ab32.txt 2>&1; cat $O/ab32.txt
for b in 1 5; do AB_N=34 AB_D=20 AB_BEAM=$b timeout 900 python tools/ab_step.py 1 $B | sed "s/^/beam$b /"; done > $O/ab34.txt 2>&1; cat $O/ab34.txt
timeout 1500 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py -x -q > $O/pytest.log 2>&1; tail -2 $O/pytest.log
