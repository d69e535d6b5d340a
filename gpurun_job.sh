python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests/test_gpu_multiproc.py -m gpu -x -q 2>&1 | tail -2
