#!/bin/bash
mkdir -p gpurun_out
timeout 300 python tools/probe_box.py > gpurun_out/probe.log 2>&1
timeout 900 python tools/k1_sweep.py run 8 > gpurun_out/sweep6.log 2>&1
timeout 900 python bench.py --shape 13B --blocks 12 --residency host --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/bench_host13b.log 2>&1
timeout 900 python bench.py --shape 13B --blocks 12 --residency host --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 --max-ctas 16 > gpurun_out/bench_host13b_mc16.log 2>&1
echo done
