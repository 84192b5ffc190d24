#!/bin/bash
# HOST_COMPUTE (the paper's CPU handler) vs handler thread count on 8 x 13B blocks; each line carries the
# run's host_stream probe.   /usr/local/graft/bin/gpurun --timeout 1800 -- 'bash tools/hostcompute_sweep.sh'
mkdir -p gpurun_out; : > gpurun_out/hc_sweep.jsonl
for rep in 1 2; do for th in ${THREADS:-0 15 14}; do
  r=$(timeout 600 python bench.py --shape 13B --residency hostcompute --blocks 8 --steps 3 --warmup 3 --host-threads $th --no-e2e --no-cpu-baseline --overlap-sweep 0 --overlap-host-sweep 0 2>/dev/null | tail -n 1)
  python -c "import json,sys; d=json.loads(sys.argv[1]); r=d['roofline']; print(json.dumps({'threads':$th,'gparams':d['value']/1e9,'gbs':r['achieved'],'peak':r['peak'],'frac':r['frac'],'sched':'${SCHED:-dynamic}'}))" "$r" >> gpurun_out/hc_sweep.jsonl
done; done
