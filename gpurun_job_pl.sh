O=gpurun_out/e2e; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_boundary.py -q > $O/pytest.log 2>&1; tail -3 $O/pytest.log
timeout 900 python bench.py --no-cpu-baseline > $O/bench.json 2> $O/bench.err; tail -1 $O/bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e'])"
