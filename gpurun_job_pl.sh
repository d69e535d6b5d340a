O=gpurun_out/m64; mkdir -p $O
V=paper_conf_sc_markidis23_b200/_variants
for L in cur m64 cur m64; do for T in 13 12; do SVB200_LIB=$PWD/$V/libsvb200_$L.so timeout 600 python bench.py --precision 64 --max-fused 1 --no-sweep --no-cpu-baseline --steps 3 --warmup 2 --block-bits $T 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$L', $T, round(d['value']*1e3,2), d['config']['passes_per_step'], round(d['roofline']['hbm']['frac'],3))"; done; done > $O/ab.txt 2>&1; cat $O/ab.txt
SVB200_LIB=$PWD/$V/libsvb200_m64.so timeout 900 python -m pytest tests/test_gpu_fp64.py -q > $O/pytest.log 2>&1; tail -3 $O/pytest.log
