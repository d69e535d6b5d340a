python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 600 python tools/tc_check.py
timeout 300 python tools/prof_apply.py 30 5 h5 h6 l6 2>&1
SVB200_TC=simt timeout 300 python tools/prof_apply.py 30 3 h6 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:apply_tci -s 1 -c 1 -o gpurun_out/prof_tci6 python tools/prof_apply.py 30 1 h6 > /dev/null 2>&1
