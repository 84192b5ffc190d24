# Same-box A/B of two libratel builds on the full bench workload (13B, 41 blocks).
mkdir -p gpurun_out
for r in 1 2 3; do for v in w16s4 w8s6; do
  RATEL_LIB=build/variants/libratel_$v.so timeout 600 python bench.py --steps 20 --no-e2e --no-cpu-baseline --overlap-sweep 0 \
    --overlap-host-sweep 0 2>/dev/null | tail -n 1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(json.dumps({'lib': '$v', 'round': $r, 'value': d['value'], 'k1_gbs': d['roofline']['achieved'], 'sm_mhz': d['clocks'].get('sm_mhz')}))" >> gpurun_out/ab.jsonl
done; done
