#!/bin/bash
# ring graphs: local-map projection serial (default) vs forked beside the extraction, K = 20 / 200.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
  for K in 20 200; do
    for F in 0 2; do
      timeout 600 python bench.py --steps $K --warmup 5 --fork-project $F --no-cpu-baseline > $OUT/fp_${K}_$F.json 2> /dev/null
      python -c "
import json; d=json.loads(open('$OUT/fp_${K}_$F.json').read().strip().splitlines()[-1])
print('K=$K fork=$F', round(d['value']), 'steady', round((d.get('steady_state') or {}).get('value') or 0), 'p50', round(d['latency_ms']['p50'],4), 'iso', round(d['latency_ms']['isolated_tick_ms'],4))"
    done
  done
done
