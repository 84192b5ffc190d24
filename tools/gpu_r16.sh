#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python tools/overlap_bench.py --shape 70B --blocks 3 --residency host --ring 0 --tokens 16384 65536 98304 --max-ctas 16 0 --steps 2 > gpurun_out/overlap_host70b.log 2>&1
echo done
