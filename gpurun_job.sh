python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
for F in 4 5; do timeout 300 python bench.py --max-fused $F --no-cpu-baseline --steps 5 --warmup 3 2>&1 | tail -1; done
timeout 300 python bench.py --qubits 32 --depth 20 --max-fused 5 --no-cpu-baseline --steps 3 --warmup 3 2>&1 | tail -1
