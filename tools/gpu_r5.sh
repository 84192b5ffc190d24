#!/bin/bash
mkdir -p gpurun_out
./build/stream_probe > gpurun_out/stream_probe.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.log 2>&1
echo done
