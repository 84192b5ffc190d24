#!/bin/bash
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:adam_update -s 4 -c 1 -o gpurun_out/k1_tma_full python bench.py --blocks 4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_tma.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1
timeout 600 python bench.py --shape 30B --blocks 12 --clip 1.0 --no-e2e --no-cpu-baseline > gpurun_out/bench_clip30b.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_clip.csv python bench.py --shape 30B --blocks 4 --clip 1.0 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_clip.log 2>&1
timeout 900 python bench.py --shape 70B --blocks 3 --residency host --steps 3 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/bench_host70b.log 2>&1
echo done
