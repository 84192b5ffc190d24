# Pinned-host residency: in-place update over the host link (RATEL_STAGING_ZERO_COPY) vs the tile ring.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "zero_copy or pinned_host" > gpurun_out/zc_tests.log 2>&1
for st in pipelined zero_copy; do for mc in 0 64 16; do
  if [ $st = pipelined ] && [ $mc != 0 ]; then continue; fi
  timeout 600 python bench.py --residency host --blocks 8 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline --overlap-sweep 0 \
     --overlap-host-sweep 0 --staging $st --max-ctas $mc 2>/dev/null | tail -n 1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(json.dumps({'staging': '$st', 'max_ctas': $mc, 'value': d['value'], 'ms': d['ms_per_step'], 'link_gbs': 24*d['value']/1e9, 'clocks': d['clocks']}))" >> gpurun_out/zc_bench.jsonl
done; done
for mc in 0 32; do
  timeout 900 python tools/overlap_bench.py --residency host --granularity tensor --blocks 8 --ring 3 --tokens 131072 \
      --max-ctas $mc --zero-copy --schedules bwd opt ago >> gpurun_out/zc_ovl.jsonl 2>> gpurun_out/zc.err
done
