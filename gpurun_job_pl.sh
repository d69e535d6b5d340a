O=gpurun_out/mr; mkdir -p $O
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29655 bench.py --gpus 2 --qubits 28 --depth 14 --steps 2 --warmup 1 > $O/b2.json 2> $O/b2.err; tail -1 $O/b2.json | cut -c1-700; tail -3 $O/b2.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29656 bench.py --gpus 4 --qubits 28 --depth 20 --steps 2 --warmup 1 > $O/b4.json 2> $O/b4.err; tail -1 $O/b4.json | cut -c1-700; tail -3 $O/b4.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29657 bench.py --impl reference --gpus 2 --steps 3 --warmup 1 > $O/r2.json 2> $O/r2.err; tail -1 $O/r2.json | cut -c1-300
