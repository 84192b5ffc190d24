# Pinned-host AGO (per-tensor hand-off, 8 x 13B blocks, 128K tokens): tile-update kernel footprint vs exposure.
mkdir -p gpurun_out
for te in 16777216 67108864; do for k in 0 2; do for mc in 0 16 4; do
  timeout 600 python tools/overlap_bench.py --residency host --granularity tensor --blocks 8 --ring 3 --tokens 131072 \
      --max-ctas $mc --k1-kernel $k --tile-elems $te --schedules bwd opt ago >> gpurun_out/host_sweep.jsonl 2>> gpurun_out/host_sweep.err
done; done; done
