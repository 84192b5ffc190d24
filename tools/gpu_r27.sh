#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -m gpu -q -rf -k "max_ranges or clip_adam_l2" > gpurun_out/pytest_new.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:adam_update -s 4 -c 1 -o gpurun_out/k1_tma_full python bench.py --blocks 4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_tma.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/ncu_launch_bench.log 2>&1
echo done
