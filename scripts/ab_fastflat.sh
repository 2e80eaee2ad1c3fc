#!/bin/bash
# FAST grid order (host switch SS_FAST_FLAT, read at ss_create): 0 = 2-D (band, frame) grid in
# longest-first band order, 1 = flat band-major (the order holds across frames), 2 = flat with
# level 0's bands first (they do not wait for the pyramid).  c2, K = 200 and K = 20.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
echo "$(timeout 600 python -m pytest tests -m gpu -q -x -k 'launch_layouts' -p no:cacheprovider 2>&1 | tail -1)"
for v in ${VARIANTS:-0 1 2 0 1 2}; do
  for K in 200 20; do
    SS_FAST_FLAT=$v timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/ff.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/ff.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  [$v] K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', round(k['fast'],1), 'frac', round(d['roofline']['frac'],3), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
