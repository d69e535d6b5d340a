O=gpurun_out/mono; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py tests/test_gpu_boundary.py -x -q > $O/pytest.log 2>&1; tail -3 $O/pytest.log
V=paper_conf_sc_markidis23_b200/_variants
AB_WL=sycamore AB_F=1 AB_PIN=3 timeout 900 python tools/ab_step.py 2 $V/libsvb200_beam5.so $V/libsvb200_mono.so > $O/syc1.txt 2>&1; cat $O/syc1.txt
AB_WL=sycamore AB_F=1 timeout 900 python tools/ab_step.py 1 $V/libsvb200_beam5.so $V/libsvb200_mono.so > $O/syc1p4.txt 2>&1; cat $O/syc1p4.txt
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; tail -1 $O/bench.json | cut -c1-300
timeout 900 python bench.py --qubits 30 --depth 14 --workload sycamore --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 > $O/syc.json; cut -c1-250 $O/syc.json
