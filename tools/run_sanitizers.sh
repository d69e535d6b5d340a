#!/bin/bash
# compute-sanitizer over tools/sanitize_cases.py (single process: rpj, apply_rpass,
# apply_pass, per-gate SIMT / int8 tcgen05 tile loops, exchange, sampler, fp64) and
# over the multi-process sharded mode (2 ranks: device barrier over IPC-mapped flag
# words, P2P exchange, merge kernels).  usage: bash tools/run_sanitizers.sh <outdir>
OUT=${1:-gpurun_out}
mkdir -p $OUT
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_cases.py > $OUT/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?: $(grep -E 'ERROR SUMMARY|SANITIZE_CASES' $OUT/sanitize_$tool.txt | tr '\n' ' ')"
done
for tool in memcheck synccheck; do
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29571 \
    --no-python compute-sanitizer --tool $tool --print-limit 50 python tools/mp_check.py 14 > $OUT/sanitize_mp_$tool.txt 2>&1
  echo "mp $tool rc=$?: $(grep -E 'ERROR SUMMARY|MP_OK|MP_FAIL' $OUT/sanitize_mp_$tool.txt | tr '\n' ' ')"
done
