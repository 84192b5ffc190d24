#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --blocks 6 --sim-comm-none --no-cpu-baseline --e2e-blocks 2 > gpurun_out/bench_sim2.log 2>&1
echo "rc=$?" >> gpurun_out/bench_sim2.log
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 --oracle-sample 4000000 > gpurun_out/bench_ref2.log 2>&1
echo "rc=$?" >> gpurun_out/bench_ref2.log
echo done
