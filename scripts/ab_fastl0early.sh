#!/bin/bash
# FAST level-0 CTAs skipping the dependency wait (run beside the pyramid): c2 K=200 / K=20 + c3.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider 2>&1 | tail -1
for rep in 1 2; do
  for K in 200 20; do
    timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/l0e_$K.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/l0e_$K.json').read().strip().splitlines()[-1])
print('K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'p50', round(d['latency_ms']['p50'],4), 'e2e', round(d['e2e']['value']))"
  done
done
timeout 600 python bench.py --config c3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c3', round(d['value']), round(d['e2e']['value']))"
