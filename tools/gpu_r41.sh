#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python tools/overlap_bench.py --tokens 8192 32768 --max-ctas 0 8 12 16 24 --carveout --schedules bwd ago --steps 2 > gpurun_out/overlap_carveout.log 2>&1
echo done
