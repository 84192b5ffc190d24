#!/bin/bash
# Hybrid residency: fraction f of each 13B block GPU-streamed (pinned-host tile ring, PCIe-bound) and the
# rest updated by the CPU handler (HOST_COMPUTE, host-DRAM-bound), both handed off at the block's gradient.
#   /usr/local/graft/bin/gpurun --timeout 2400 -- 'bash tools/hybrid_sweep.sh'
mkdir -p gpurun_out; : > gpurun_out/hybrid.jsonl
for f in ${FRACS:-0 0.2 0.3 0.4 0.5 0.6 1}; do
  timeout 600 python bench.py --shape 13B --residency hybrid --hybrid-gpu-frac $f --blocks 8 --steps 3 --warmup 3 \
      --no-e2e --no-cpu-baseline --overlap-sweep 0 --overlap-host-sweep 0 2>>gpurun_out/hybrid.err | tail -n 1 >> gpurun_out/hybrid.jsonl
done
