#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_api_gpu.py -m gpu -q -rf -x > gpurun_out/pytest_api.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.log 2>&1
echo done
