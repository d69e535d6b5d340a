python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests -q -m gpu 2>&1 | tail -6
for F in 2 4 5; do timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --max-fused $F --precision 64 --samples 100000 | cut -c1-250; done
