#!/bin/bash
mkdir -p gpurun_out
timeout 900 python tools/k1_sweep.py run 8 > gpurun_out/sweep.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
echo done
