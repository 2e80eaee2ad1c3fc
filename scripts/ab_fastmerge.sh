#!/bin/bash
# FAST as one launch after the pyramid (default) vs level 0 beside the pyramid (SS_FAST_SPLIT=1).
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -q -x -k "parity or coverage or track" -p no:cacheprovider 2>&1 | tail -2
for rep in 1 2; do
  for S in 0 1; do
    for C in c2 c3; do
      SS_FAST_SPLIT=$S timeout 600 python bench.py --config $C --no-cpu-baseline > $OUT/fm_${S}_${C}_$rep.json 2> /dev/null
      python -c "
import json; d=json.loads(open('$OUT/fm_${S}_${C}_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('split=$S $C', round(d['value']), 'steady', round(d['steady_state']['value']), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), d['roofline']['kernel'], round(d['roofline']['frac'],3), {a: round(b,1) for a,b in k.items() if 'fast' in a})"
    done
  done
done
