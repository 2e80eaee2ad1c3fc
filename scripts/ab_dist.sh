#!/bin/bash
# quadtree (216 KB smem, 1024-thread CTAs) vs grid top-N (1024 threads, ~40 KB smem) on c2.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2 3; do
  for D in quadtree grid; do
    timeout 600 python bench.py --dist $D --no-cpu-baseline > $OUT/dist_${D}_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/dist_${D}_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('$D', round(d['value']), 'steady', round(d['steady_state']['value']), 'dist', round(k.get('distribute_l0',0),1), round(k.get('distribute_l1plus',0),1), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
