#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py --shape 30B --blocks 12 --clip 1.0 --no-e2e --no-cpu-baseline > gpurun_out/bench_clip30b.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:grad_sumsq --csv --log-file gpurun_out/launches_k2.csv python bench.py --shape 30B --blocks 4 --clip 1.0 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_clip.log 2>&1
echo done
