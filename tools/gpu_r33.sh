#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
timeout 1500 python tools/overlap_bench.py --shape 13B --blocks 8 --residency host --ring 0 --tokens 98304 --max-ctas 16 --schedules bwd opt ago deferred naive --steps 2 --timeline > gpurun_out/overlap_tl2.log 2>&1
timeout 900 python bench.py --shape 13B --blocks 8 --residency host --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 --depth 8 > gpurun_out/bench_host_d8.log 2>&1
echo done
