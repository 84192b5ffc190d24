#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
timeout 1500 python tools/overlap_bench.py --shape 13B --blocks 8 --residency host --ring 0 --tokens 32768 98304 --max-ctas 16 --schedules bwd opt ago deferred naive --steps 2 > gpurun_out/overlap_host13b_v3.log 2>&1
timeout 1500 python tools/overlap_bench.py --shape 13B --blocks 8 --residency hostcompute --ring 0 --tokens 32768 98304 --max-ctas 0 --schedules bwd opt ago deferred --steps 2 > gpurun_out/overlap_hostcompute_v3.log 2>&1
echo done
