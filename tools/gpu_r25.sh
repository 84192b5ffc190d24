#!/bin/bash
mkdir -p gpurun_out
for v in ldg rel1 rel3 rel4; do
  RATEL_LIB=build/variants/libratel_$v.so timeout 900 compute-sanitizer --tool racecheck --kernel-name kns=ratel --print-limit 4 python tools/sanitize_run.py > gpurun_out/racecheck_$v.log 2>&1
done
echo done
