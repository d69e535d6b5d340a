O=gpurun_out/czf2; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py tests/test_gpu_fullsize.py tests/test_gpu_fp64.py -x -q > $O/pytest.log 2>&1; tail -3 $O/pytest.log
