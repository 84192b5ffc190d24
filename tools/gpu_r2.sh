#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_parity_gpu.py -m gpu -x -q -k "adam_l2" > gpurun_out/t_l2.log 2>&1
timeout 300 python -X faulthandler -m pytest tests/test_parity_gpu.py -m gpu -x -q -s -k "overlapped" > gpurun_out/t_ovl.log 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py -m gpu -q -rf --deselect tests/test_parity_gpu.py::test_overlapped_with_backward_stream > gpurun_out/t_rest.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:adam_update -s 4 -c 2 -o gpurun_out/k1_full python bench.py --blocks 4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
echo done
