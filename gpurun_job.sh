python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests/test_gpu_multiproc.py -q -x 2>&1 | tail -30
timeout 900 python -m pytest tests -q -m gpu 2>&1 | tail -3
timeout 600 python bench.py --steps 5 --warmup 3 --cpu-seconds 15 2>&1 | tail -1 > gpurun_out/bench_r1.json; cat gpurun_out/bench_r1.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --samples 100000 > gpurun_out/ncu_launch_bench.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:apply_high -s 2 -c 1 -o gpurun_out/prof_bench_h4 python tools/prof_apply.py 30 2 h4 > /dev/null 2>&1
ncu -i gpurun_out/prof_bench_h4.ncu-rep --page raw --csv > gpurun_out/prof_bench_h4_raw.csv 2>/dev/null
ls -la gpurun_out
