#!/bin/bash
# FAST launch bounds: 3 CTAs per SM (80 registers, default) vs 4 (64 registers, spills), c2 bench.
set -u
OUT=gpurun_out; mkdir -p $OUT
for M in 3 4; do
  SS_NVCC_EXTRA="-DSS_FAST_MINB=$M" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  [ $M = 3 ] && { timeout 600 python -m pytest tests -m gpu -q -x -k "parity" -p no:cacheprovider 2>&1 | tail -1; }
  for rep in 1 2; do
    timeout 600 python bench.py --no-cpu-baseline > $OUT/mb_$M.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/mb_$M.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('minb=$M', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', round(k['fast'],1), 'frac', round(d['roofline']['frac'],3), 'iso', round(d['latency_ms']['isolated_tick_ms'],4))"
  done
done
