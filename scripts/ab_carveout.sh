#!/bin/bash
# One fixed shared-memory carveout on the extraction kernels (SS_CARVEOUT percent) vs the driver's choice, c2.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
  for C in none 100; do
    if [ $C = none ]; then unset SS_CARVEOUT; else export SS_CARVEOUT=$C; fi
    timeout 600 python bench.py --steps 200 --warmup 5 --no-cpu-baseline > $OUT/co_$C.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/co_$C.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('carveout=$C', round(d['value']), 'steady', round(d['steady_state']['value']), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), {a: round(b,1) for a,b in k.items()})"
  done
done
