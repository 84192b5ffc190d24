#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_sharded_gpu.py tests/test_abi_cpu.py -q -rf -x > gpurun_out/pytest_sharded.log 2>&1
timeout 1800 python tools/overlap_bench.py --shape 13B --blocks 12 --residency host --ring 0 --tokens 32768 98304 --max-ctas 16 --steps 2 > gpurun_out/overlap_host13b.log 2>&1
echo done
