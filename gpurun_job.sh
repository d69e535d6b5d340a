python -c "import __graft_entry__ as g; g.build()" > /dev/null
python tools/norm_drift.py 18 4 20
python tools/norm_drift.py 18 5 20
timeout 300 python tools/prof_apply.py 30 5 h4 l4 q0 h5 l5 2>&1
