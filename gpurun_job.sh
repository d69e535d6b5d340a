python -c "import __graft_entry__ as g; g.build()" > /dev/null
SVB200_TC=i8 timeout 600 python tools/tc_check.py
SVB200_TC=i8 timeout 300 python tools/prof_apply.py 30 5 h4 l4 q0 h5 l5 h6 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:apply_tci -s 1 -c 1 -o gpurun_out/prof_tci python tools/prof_apply.py 30 1 h5 > /dev/null 2>&1
