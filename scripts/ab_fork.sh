#!/bin/bash
# A/B: local-map projection forked off the critical path in the ring graphs (one gpurun call).
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
for F in 0 1; do
  for S in 20 200; do
    timeout 600 python bench.py --fork-project $F --steps $S --no-cpu-baseline > $OUT/fork_${F}_${S}_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/fork_${F}_${S}_$rep.json').read().strip().splitlines()[-1])
print('fork=$F steps=$S', round(d['value']), 'steady', round((d['steady_state'] or {}).get('value', 0)), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
done
