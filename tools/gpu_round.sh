#!/bin/bash
# Full evidence collection on one B200 (run via gpurun):
#   /usr/local/graft/bin/gpurun --timeout 3600 -- 'bash tools/gpu_round.sh'
# Results land in gpurun_out/; copy what should be judged into profiles/.
set -u
mkdir -p gpurun_out
timeout 300  python tools/probe_box.py                  > gpurun_out/probe.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -rf       > gpurun_out/pytest_gpu.log 2>&1
timeout 300  python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1200 python bench.py                            > gpurun_out/bench.log 2>&1
timeout 900  python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.log 2>&1
# launch list of the bench command (cold-cache, serialised: compare shares)
timeout 900  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
             --csv --log-file gpurun_out/launches.csv \
             python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --overlap-sweep 0 --overlap-host-sweep 0 > gpurun_out/ncu_launch.log 2>&1
# one full capture of K1 on a 13B block
timeout 900  ncu --set full --clock-control none --import-source on -k regex:adam_update -s 4 -c 1 -o gpurun_out/k1_full \
             python bench.py --blocks 4 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --overlap-sweep 0 --overlap-host-sweep 0 > gpurun_out/ncu_full.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --kernel-name kns=ratel --print-limit 10 python tools/sanitize_run.py \
              > gpurun_out/sanitizer_$tool.log 2>&1
done
echo done
