#!/bin/bash
# The trigger points re-checked at 8 ticks in flight: (distribution phase, pyramid level) =
# (8, 3) default / (0, 3) / (8, 0), K = 200 and K = 20, two interleaved rounds.
set -u
OUT=gpurun_out; mkdir -p $OUT
for rep in 1 2; do
  for v in "8 3" "0 3" "8 0"; do
    set -- $v
    SS_NVCC_EXTRA="-DSS_DIST_TRIGGER=$1 -DSS_PYR_TRIGGER=$2" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
    for K in 200 20; do
      timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/t8.json 2> /dev/null
      python -c "
import json; d=json.loads(open('$OUT/t8.json').read().strip().splitlines()[-1])
print('dist=$1 pyr=$2 K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4))"
    done
  done
done
