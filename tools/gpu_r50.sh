#!/bin/bash
mkdir -p gpurun_out
timeout 900 python bench.py --shape 13B --blocks 8 --residency hostcompute --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/bench_hc_fp64.log 2>&1
RATEL_LIB=build/variants/libratel_hostfp32.so timeout 900 python bench.py --shape 13B --blocks 8 --residency hostcompute --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/bench_hc_fp32.log 2>&1
RATEL_LIB=build/variants/libratel_hostfp32.so timeout 900 python -m pytest tests/test_parity_gpu.py -m gpu -q -k host_compute > gpurun_out/pytest_hc32.log 2>&1
echo done
