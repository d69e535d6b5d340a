mkdir -p gpurun_out/spec
timeout 900 python -m pytest tests/test_gpu_jit.py -q > gpurun_out/spec/jit.log 2>&1; tail -5 gpurun_out/spec/jit.log
V=paper_conf_sc_markidis23_b200/_variants
for pin in 3 4 5; do echo "pin $pin"; AB_PIN=$pin timeout 900 python tools/ab_step.py 3 $V/libsvb200_base.so $V/libsvb200_ring.so $V/libsvb200_pf.so $V/libsvb200_m4.so; done 2>&1 | tee gpurun_out/spec/ab.log
