mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1800 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log | cut -c1-200
bash tools/run_configs.sh gpurun_out/configs.jsonl > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_f1.csv python bench.py --max-fused 1 --no-sweep --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1; echo ncu rc $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:apply_rpass -s 5 -c 1 -o gpurun_out/rpass_full python bench.py --max-fused 1 --no-sweep --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo ncu rc $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:apply_rpass -s 0 -c 1 -o gpurun_out/rpass_full_p0 python bench.py --max-fused 1 --no-sweep --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_full0.log 2>&1; echo ncu rc $?
SVB200_RPASS_DEBUG=1 timeout 300 python bench.py --max-fused 1 --no-sweep --steps 1 --warmup 0 --no-cpu-baseline 2>gpurun_out/rpdbg.txt >/dev/null
