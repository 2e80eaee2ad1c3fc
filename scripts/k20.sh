#!/bin/bash
# Short (driver-like, K = 20) vs long bench runs of the default config, a few repetitions.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2 3; do
  for S in 20 200; do
    timeout 600 python bench.py --steps $S --warmup 3 --no-cpu-baseline > $OUT/k_${S}_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/k_${S}_$rep.json').read().strip().splitlines()[-1])
print('steps=$S', round(d['value']), 'steady', round((d['steady_state'] or {}).get('value', 0)), 'p50', round(d['latency_ms']['p50'],4), 'ms', round(d['ms_per_step'],4))"
  done
done
