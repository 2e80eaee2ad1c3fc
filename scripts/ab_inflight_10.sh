#!/bin/bash
# Ticks in flight at HEAD: --inflight 8 (default) / 10, the driver's K = 20 command three
# times each (interleaved) and K = 200 once each.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2 3; do
  for P in 8 10; do
    timeout 600 python bench.py --inflight $P --steps 20 --warmup 5 --no-cpu-baseline > $OUT/ih.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/ih.json').read().strip().splitlines()[-1])
print('P=$P K=20', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
for P in 8 10; do
  timeout 600 python bench.py --inflight $P --steps 200 --warmup 5 --no-cpu-baseline > $OUT/ih.json 2> /dev/null
  python -c "
import json; d=json.loads(open('$OUT/ih.json').read().strip().splitlines()[-1])
print('P=$P K=200', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4))"
done
