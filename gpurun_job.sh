python -c "import __graft_entry__ as g; g.build()" > /dev/null
python tools/prof_apply.py 30 5 h1 l1 h2 l2 h3 l3 h4 l4 l4b q0 h5 l5 h6 l6 2>&1
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -4
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1
