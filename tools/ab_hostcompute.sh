#!/bin/bash
# Same-box A/B of the CPU handler's P16 staging store: non-temporal (default) vs plain, 8 x 13B blocks,
# plus the hybrid residency with each build.
mkdir -p gpurun_out; : > gpurun_out/ab_hc.jsonl
for r in 1 2 3; do for v in nt nont; do for res in hostcompute hybrid; do
  RATEL_LIB=build/variants_hc/libratel_$v.so timeout 600 python bench.py --shape 13B --residency $res --blocks 8 --steps 3 --warmup 3 \
    --no-e2e --no-cpu-baseline --overlap-sweep 0 --overlap-host-sweep 0 2>/dev/null | tail -n 1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print(json.dumps({'lib': '$v', 'residency': '$res', 'round': $r, 'gparams': d['value']/1e9, 'host_dram_gbs': r['host_dram']['achieved'], 'probe_gbs': r['host_dram']['peak']}))" >> gpurun_out/ab_hc.jsonl
done; done; done
