python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -4
timeout 900 python tools/micro_bench.py 2>&1 | grep -E "small"
timeout 600 python bench.py --qubits 12 --depth 14 --max-fused 0 --steps 20 --warmup 3 --cpu-seconds 5 | cut -c1-400
