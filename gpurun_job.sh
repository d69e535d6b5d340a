python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -4
timeout 900 python tools/micro_bench.py gpurun_out/micro_r1b.json 2>&1 | grep -E "sample|exchange"
