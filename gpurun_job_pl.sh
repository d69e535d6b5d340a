O=gpurun_out/p0b; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_jit.py tests/test_gpu_circuit.py tests/test_gpu_fullsize.py -x -q > $O/pytest.log 2>&1; tail -2 $O/pytest.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; tail -1 $O/bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline']['alu']['frac'], d['roofline']['pass_floor']['frac'], d['config']['execution'][-45:])"
