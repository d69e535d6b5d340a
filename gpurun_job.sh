mkdir -p gpurun_out/comm
timeout 1200 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py -q -x > gpurun_out/comm/t.log 2>&1; tail -3 gpurun_out/comm/t.log
V=paper_conf_sc_markidis23_b200/_variants
for pin in 3 4; do echo "pin $pin"; AB_PIN=$pin timeout 900 python tools/ab_step.py 2 $V/libsvb200_base.so $V/libsvb200_ring.so; done 2>&1 | tee gpurun_out/comm/ab.log
for v in base ring; do echo "32q $v"; AB_N=32 AB_D=20 SVB200_LIB=$V/libsvb200_$v.so timeout 600 python tools/ab_step.py 1 $V/libsvb200_$v.so; done
