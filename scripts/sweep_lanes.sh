#!/bin/bash
# WINDOW-matcher lanes-per-query sweep on a config (one gpurun call).  Usage: bash scripts/sweep_lanes.sh [config]
set -u
OUT=gpurun_out; mkdir -p $OUT
C=${1:-c2}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for WG in ${LANES:-0 1 2 4 8}; do
  timeout 600 python bench.py --config $C --match-lanes $WG --no-cpu-baseline > $OUT/lanes_${C}_$WG.json 2> $OUT/lanes_${C}_$WG.err
  python -c "
import json; d=json.loads(open('$OUT/lanes_${C}_$WG.json').read().strip().splitlines()[-1])
print('lanes=$WG', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4), 'mw', round(d['kernels_us']['match_window'],1))"
done
