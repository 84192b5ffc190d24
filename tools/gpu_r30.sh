#!/bin/bash
mkdir -p gpurun_out
for th in 0 8; do
timeout 900 python bench.py --shape 13B --blocks 8 --residency hostcompute --host-threads $th --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/bench_hostcompute_t$th.log 2>&1
done
timeout 1500 python tools/overlap_bench.py --shape 13B --blocks 8 --residency hostcompute --ring 0 --tokens 32768 98304 --max-ctas 0 --schedules bwd opt ago deferred --steps 2 > gpurun_out/overlap_hostcompute.log 2>&1
echo done
