#!/bin/bash
# Run bench.py on every BASELINE.json config that fits one GPU (plus the
# NEXT-1/NEXT-4 variants); one JSON line each.  usage: bash tools/run_configs.sh <out.jsonl>
OUT=${1:-gpurun_out/configs.jsonl}
: > $OUT
run() { timeout 1200 python bench.py "$@" 2>/dev/null | tail -1 >> $OUT; tail -1 $OUT | cut -c1-160; }
run --qubits 12 --depth 14 --max-fused 0 --steps 20 --warmup 3 --cpu-seconds 5 --no-sweep
run --qubits 30 --depth 14 --steps 5 --warmup 3 --no-cpu-baseline
run --qubits 32 --depth 20 --steps 3 --warmup 3 --no-cpu-baseline
run --qubits 34 --depth 20 --max-fused 1 --steps 2 --warmup 2 --no-cpu-baseline --no-sweep
run --qubits 30 --depth 14 --workload sycamore --steps 5 --warmup 3 --no-cpu-baseline
run --qubits 30 --depth 14 --precision 64 --max-fused 1 --steps 3 --warmup 2 --no-cpu-baseline --no-sweep
run --qubits 30 --depth 14 --precision 64 --max-fused 4 --steps 3 --warmup 2 --no-cpu-baseline --no-sweep
run --qubits 30 --depth 14 --precision 64 --max-fused 1 --steps 3 --warmup 2 --no-cpu-baseline --no-sweep --pass-search 1
