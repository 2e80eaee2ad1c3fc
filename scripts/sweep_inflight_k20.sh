#!/bin/bash
# K = 20 (the driver's run) vs ticks in flight P, two reps each, c2.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
  for P in 4 5 6 10 20; do
    timeout 600 python bench.py --steps 20 --warmup 5 --inflight $P --no-cpu-baseline > $OUT/k20_$P.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/k20_$P.json').read().strip().splitlines()[-1])
print('K=20 P=$P', round(d['value']), 'p50', round(d['latency_ms']['p50'],4), 'e2e', round(d['e2e']['value']))"
  done
done
for P in 5 8; do
  timeout 600 python bench.py --steps 200 --warmup 5 --inflight $P --no-cpu-baseline > $OUT/k200_$P.json 2> /dev/null
  python -c "
import json; d=json.loads(open('$OUT/k200_$P.json').read().strip().splitlines()[-1])
print('K=200 P=$P', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4))"
done
