# AGO overlap (device-resident, 8 x 13B blocks): backward stream priority, grad ring depth, update-kernel variant.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "cta_tiles or max_ctas or k1_kernel" > gpurun_out/yield_tests.log 2>&1
for pr in -2 0; do for ring in 3 8; do for k in 0 2; do
  timeout 600 python tools/overlap_bench.py --residency device --blocks 8 --ring $ring --tokens 8192 --max-ctas 0 --schedules bwd opt ago --k1-kernel $k --bwd-priority $pr >> gpurun_out/yield_ovl2.jsonl 2>> gpurun_out/yield.err
done; done; done
