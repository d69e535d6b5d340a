mkdir -p gpurun_out
for M in 4 5; do SVB200_RPASS_M=$M timeout 600 python -m pytest tests/test_gpu_circuit.py -m gpu -x -q -k blocked 2>&1 | tail -1; done
for F2 in 0 1; do for M in 4 5; do for F in 1 2; do
SVB200_RPASS_F2=$F2 SVB200_RPASS_M=$M timeout 300 python bench.py --max-fused $F --block-bits 12 --steps 3 --warmup 3 --no-sweep --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('F2',$F2,'M',$M,'T',12,'F',$F, d['value'])"
done; done; done
for M in 4 5; do
SVB200_RPASS_M=$M timeout 600 ncu --set full --clock-control none --import-source on -k regex:apply_rpass -s 3 -c 1 -o gpurun_out/rpass12m${M}f2 python bench.py --max-fused 2 --block-bits 12 --steps 1 --warmup 3 --no-sweep --no-cpu-baseline > gpurun_out/ncu_pass.log 2>&1; echo ncu rc $?
done
