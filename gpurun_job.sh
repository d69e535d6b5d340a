python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests/test_gpu_circuit.py -q -x -k "blocked" 2>&1 | grep -E "Error|error|assert" | head -10
timeout 600 ncu --set full --import-source on --clock-control none -k regex:apply_pass -s 3 -c 1 -o gpurun_out/prof_pass python bench.py --steps 1 --warmup 1 --no-cpu-baseline --max-fused 3 --block-bits 12 --samples 1000 > /dev/null 2>&1
ls gpurun_out/
