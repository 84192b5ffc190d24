#!/bin/bash
mkdir -p gpurun_out
for arm in before after; do
timeout 900 python bench.py --shape 13B --blocks 12 --residency host --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 --arm $arm > gpurun_out/bench_host13b_$arm.log 2>&1
done
timeout 1200 python tools/overlap_bench.py --shape 13B --blocks 12 --residency host --ring 0 --tokens 8192 --max-ctas 16 --schedules bwd opt ago --steps 2 > gpurun_out/overlap_host13b_b.log 2>&1
timeout 1200 python tools/overlap_bench.py --shape 13B --blocks 12 --residency host --ring 3 --tokens 8192 --max-ctas 16 --schedules bwd opt ago --steps 2 > gpurun_out/overlap_host13b_c.log 2>&1
echo done
