#!/bin/bash
# e2e ticks in flight (host-memory path through ss_track_run): 8 (default) / 10 / 12, c2.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
  for E in 8 10 12; do
    timeout 600 python bench.py --e2e-inflight $E --steps 20 --warmup 5 --no-cpu-baseline > $OUT/ei.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/ei.json').read().strip().splitlines()[-1]); e=d['e2e']
print('e2e_inflight=$E', round(e['value']), 'mode', e.get('mode'), 'device', round(d['value']))"
  done
done
