#!/bin/bash
# One validation job on a B200 box: smoke, GPU suite, bench, configs, ncu
# launch list and full captures of every pass of the 30q D14 F=1 circuit in
# the bench's chosen configuration, sanitizers.
# usage: gpurun -- 'bash gpurun_job.sh <tag> [pass_search]'
T=${1:-job}
PS=${2:-1}
O=gpurun_out/$T
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; tail -5 $O/pytest.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; tail -1 $O/bench.json | cut -c1-400
if [ "${NO_CONFIGS:-0}" = 0 ]; then bash tools/run_configs.sh $O/configs.jsonl; fi
# the pass formation and run width the bench chose (for the ncu runs)
PS=$(python -c "import json,re; d=json.loads(open('$O/bench.json').read().strip().split(chr(10))[-1]); print(re.search(r'SV_OPT_PASS_SEARCH (\d)', d['config']['execution']).group(1))" 2>/dev/null || echo $PS)
PIN=$(python -c "import json,re; d=json.loads(open('$O/bench.json').read().strip().split(chr(10))[-1]); print(re.search(r'SV_OPT_PASS_PIN (\d)', d['config']['execution']).group(1))" 2>/dev/null || echo 4)
echo "ncu with pass search $PS, pin $PIN" > $O/ncu_config.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
  --log-file $O/launches.csv python bench.py --steps 2 --warmup 1 --no-sweep --no-cpu-baseline --pass-search $PS --pass-pin $PIN > $O/ncu_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:rpj -c 12 \
  -o $O/rpj_full python tools/prof_circuit.py 30 14 1 1 $PIN 1 $PS > $O/ncu_full.log 2>&1
ncu -i $O/rpj_full.ncu-rep --page raw --csv > $O/rpj_full_raw.csv 2>/dev/null
# compute-sanitizer is closed on the round-2 pool (it left GPUs needing a reset);
# the round-2 logs from before the closure are in profiles/r2_sanitize/
if [ "${SAN:-0}" = 1 ]; then bash tools/run_sanitizers.sh $O/sanitize > $O/sanitize.log 2>&1; cat $O/sanitize.log; fi
echo done
