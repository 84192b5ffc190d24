#!/bin/bash
# R7 A/B: K1 with sqrt.approx/rcp.approx (default build)
# vs IEEE __fsqrt_rn/__fdiv_rn (RATEL_K1_FASTMATH=0, build/variants/libratel_ieee.so),
# alternating rounds of the bench's main measurement on the same box.
# Build the variant first:  python -c "from paper_conf_icde_liaosyxcyww25_b200 import _build; \
#   _build.build(out='build/variants/libratel_ieee.so', defines=['RATEL_K1_FASTMATH=0'])"
OUT=${1:-gpurun_out/r7_ab.jsonl}
ROUNDS=${ROUNDS:-3}
: > "$OUT"
for r in $(seq 1 "$ROUNDS"); do
  for v in approx ieee; do
    if [ "$v" = ieee ]; then export RATEL_LIB=build/variants/libratel_ieee.so; else unset RATEL_LIB; fi
    line=$(python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --overlap-sweep 0 \
           --overlap-host-sweep 0 2>/dev/null | grep '^{')
    python - "$v" "$r" "$line" >> "$OUT" <<'PY'
import json, sys
v, r, line = sys.argv[1], int(sys.argv[2]), json.loads(sys.argv[3])
print(json.dumps({"variant": v, "round": r, "value": line["value"], "ms_per_step": line["ms_per_step"],
                  "k1_gbs": line["roofline"]["achieved"], "k1_frac": line["roofline"]["frac"],
                  "clocks": line["clocks"]}))
PY
  done
done
cat "$OUT"
