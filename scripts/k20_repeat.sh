#!/bin/bash
# The driver's bench command (--steps 20 --warmup 5) repeated on one box: the spread of the
# 20-step number (fill + drain of 6 ticks in flight inside a ~0.9 ms timed region).
set -u
OUT=gpurun_out/k20rep; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2 3 4 5 6; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > $OUT/k20_$i.json 2> /dev/null
  python -c "
import json; d=json.loads(open('$OUT/k20_$i.json').read().strip().splitlines()[-1])
print('K=20 run $i', round(d['value']), 'steady', round(d['steady_state']['value']), 'e2e', round(d['e2e']['value']), 'p50', round(d['latency_ms']['p50'],4))"
done
timeout 600 python bench.py --steps 200 --warmup 5 --no-cpu-baseline > $OUT/k200.json 2> /dev/null
python -c "
import json; d=json.loads(open('$OUT/k200.json').read().strip().splitlines()[-1])
print('K=200', round(d['value']), 'steady', round(d['steady_state']['value']), 'e2e', round(d['e2e']['value']))"
