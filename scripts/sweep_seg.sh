#!/bin/bash
# FAST segment-size sweep: SS_SEG0 (level-0 cells per CTA) / SS_SEG (levels >= 1), c2 bench.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for V in ${SEGS:-"8 8" "12 8" "8 12" "12 12" "24 8"}; do
  set -- $V
  for rep in 1 2; do
    SS_SEG0=$1 SS_SEG=$2 timeout 600 python bench.py --config ${CFG:-c2} --no-cpu-baseline > $OUT/seg_$1_$2_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/seg_$1_$2_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('seg0=$1 seg=$2 ${CFG:-c2}', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', [round(v,1) for n,v in k.items() if n.startswith('fast')], 'p50', round(d['latency_ms']['p50'],4), [round(r['frac'],3) for r in d['rooflines'] if r['kernel'].startswith('fast')])"
  done
done
