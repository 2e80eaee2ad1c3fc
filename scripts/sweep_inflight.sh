#!/bin/bash
# Ticks-in-flight sweep of the c2 bench (one gpurun call).  Usage: bash scripts/sweep_inflight.sh [config]
set -u
OUT=gpurun_out; mkdir -p $OUT
C=${1:-c2}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for P in ${INFLIGHT:-3 4 5 6 8}; do
  timeout 600 python bench.py --config $C --inflight $P --no-cpu-baseline > $OUT/sweep_${C}_p$P.json 2> $OUT/sweep_${C}_p$P.err
  python -c "
import json; d=json.loads(open('$OUT/sweep_${C}_p$P.json').read().strip().splitlines()[-1])
print('P=$P', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4), 'iso', round(d['latency_ms']['isolated_tick_ms'],4))"
done
