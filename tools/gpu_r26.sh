#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --kernel-name kns=ratel --print-limit 10 python tools/sanitize_run.py > gpurun_out/sanitizer_$tool.log 2>&1
done
timeout 900 python tools/k1_sweep.py run 8 > gpurun_out/sweep8.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.log 2>&1
echo done
