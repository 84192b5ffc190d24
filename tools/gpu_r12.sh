#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python tools/overlap_bench.py --tokens 2048 8192 32768 --max-ctas 0 32 > gpurun_out/overlap_13b.log 2>&1
timeout 900 python tools/overlap_bench.py --blocks 8 --ring 0 --tokens 1024 4096 16384 --max-ctas 0 32 > gpurun_out/overlap_8blk.log 2>&1
echo done
