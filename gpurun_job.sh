python -c "import __graft_entry__ as g; g.build()" > /dev/null
for v in main r2 r4 nomono main; do
  if [ $v = main ]; then L=""; else L=paper_conf_sc_markidis23_b200/_variants/libsvb200_$v.so; fi
  echo "== $v"; SVB200_LIB=$L python tools/prof_apply.py 30 5 h1 h2 h3 h4 l4 q0 h5 2>&1
done
timeout 900 python -m pytest tests -q -m gpu 2>&1 | tail -8
