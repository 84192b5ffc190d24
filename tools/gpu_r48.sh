#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -m gpu -q -rf -k "host_compute or mixed or back_to_back or record_stream" > gpurun_out/pytest_hc.log 2>&1
for th in 0 8; do
timeout 900 python bench.py --shape 13B --blocks 8 --residency hostcompute --host-threads $th --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --overlap-tokens 0 > gpurun_out/bench_hostcompute_t$th.log 2>&1
done
echo done
