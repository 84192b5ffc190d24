#!/bin/bash
mkdir -p gpurun_out
./build/stream_probe > gpurun_out/stream_probe.log 2>&1
timeout 900 python tools/k1_sweep.py run 8 > gpurun_out/sweep3.log 2>&1
echo done
