mkdir -p gpurun_out/pk
timeout 1200 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py -q -x > gpurun_out/pk/t.log 2>&1; tail -3 gpurun_out/pk/t.log
for pin in 3 4; do AB_PIN=$pin timeout 600 python tools/ab_step.py 2 paper_conf_sc_markidis23_b200/libsvb200.so; done
AB_N=32 AB_D=20 timeout 600 python tools/ab_step.py 1 paper_conf_sc_markidis23_b200/libsvb200.so
