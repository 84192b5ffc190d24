#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python tools/overlap_bench.py --tokens 8192 32768 --max-ctas 0 16 --schedules bwd opt ago --steps 2 > gpurun_out/overlap_dev_power.log 2>&1
RATEL_LIB=build/variants/libratel_ldg.so timeout 1200 python tools/overlap_bench.py --tokens 8192 --max-ctas 0 64 --schedules bwd opt ago --steps 2 > gpurun_out/overlap_dev_ldg.log 2>&1
timeout 900 python bench.py --no-cpu-baseline --overlap-tokens 0 > gpurun_out/bench_e2e.log 2>&1
echo done
