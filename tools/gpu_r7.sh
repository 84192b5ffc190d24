#!/bin/bash
mkdir -p gpurun_out
timeout 900 python tools/k1_sweep.py run 8 > gpurun_out/sweep4.log 2>&1
echo done
