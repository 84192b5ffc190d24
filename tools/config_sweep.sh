#!/bin/bash
# bench.py on the other BASELINE.json configs (N=1), one JSON line each, into gpurun_out/configs.jsonl:
#   C3 30B-shape blocks with the global clip, C4 70B-shape pinned-host, C5 175B-shape pinned-host,
#   N2 HOST_COMPUTE (the paper's CPU handler) on 13B blocks, C1 (tiny block, launch-bound).
#   /usr/local/graft/bin/gpurun --timeout 2400 -- 'bash tools/config_sweep.sh'
set -u
mkdir -p gpurun_out
out=gpurun_out/configs.jsonl
: > $out
common="--no-e2e --no-cpu-baseline --overlap-sweep 0 --overlap-host-sweep 0"
run() { timeout 900 python bench.py "$@" $common 2> gpurun_out/configs_err.log | tail -n 1 >> $out; }
run --shape 30B --blocks 12 --clip 1.0 --steps 20 --warmup 3
run --shape 70B --residency host --blocks 3 --steps 3 --warmup 3
run --shape 175B --residency host --blocks 2 --steps 3 --warmup 3
run --shape 13B --residency hostcompute --blocks 8 --steps 3 --warmup 3
run --shape c1 --steps 200 --warmup 10

# the hybrid residency (30 % GPU-streamed + 70 % CPU handler) on the C4 / C5 shapes
run --shape 70B --residency hybrid --blocks 3 --steps 3 --warmup 3
run --shape 175B --residency hybrid --blocks 2 --steps 3 --warmup 3
# per-rank HBM work of C3 at N = 8 / 4 (rank 0 of a simulated world, no collectives)
timeout 900 python tools/rank_sim.py --shape 30B --worlds 8 4 --clip 1.0 > gpurun_out/rank_sim.jsonl 2>> gpurun_out/configs_err.log
echo done
