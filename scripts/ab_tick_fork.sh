#!/bin/bash
# A/B of ss_track_tick's forked local-map projection (e2e path), SS_TICK_FORK=1 / 0, and the
# e2e in-flight depth.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
  for F in 1 0; do
    for E in 8 12; do
      SS_TICK_FORK=$F timeout 600 python bench.py --steps 50 --e2e-inflight $E --no-cpu-baseline > $OUT/tf_${F}_${E}_$rep.json 2> /dev/null
      python -c "
import json; d=json.loads(open('$OUT/tf_${F}_${E}_$rep.json').read().strip().splitlines()[-1])
e=d['e2e']; print('fork=$F e2e_inflight=$E', round(d['value']), 'e2e', round(e['value']), e['mode'], {k: round(v) for k,v in e['trials'].items()}, round(e['host_us_per_call'],1))"
    done
  done
done
