mkdir -p gpurun_out/t14
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/t14/pytest.log 2>&1; tail -15 gpurun_out/t14/pytest.log
timeout 900 python bench.py > gpurun_out/t14/bench.json 2> gpurun_out/t14/bench.err; tail -1 gpurun_out/t14/bench.json | cut -c1-600
