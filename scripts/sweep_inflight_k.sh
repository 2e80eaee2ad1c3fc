#!/bin/bash
# ticks in flight (P) vs the timed step count (K): value / steady / p50 on c2.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for K in 20 200; do
  for P in 4 5 6 8 10; do
    timeout 600 python bench.py --steps $K --warmup 5 --inflight $P --no-cpu-baseline > $OUT/ifk_${K}_$P.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/ifk_${K}_$P.json').read().strip().splitlines()[-1])
print('K=$K P=$P', round(d['value']), 'steady', round((d.get('steady_state') or {}).get('value') or 0), 'p50', round(d['latency_ms']['p50'],4), 'e2e', round(d['e2e']['value']))"
  done
done
