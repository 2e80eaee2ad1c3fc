#!/bin/bash
# Where the frame-to-frame matcher's PDL trigger sits (SS_LF_TRIGGER: 0 = its start, 1 = after pass 0's search,
# -1 = exit): the window matcher's CTAs sit resident from the trigger until O13 ends.
set -u
OUT=gpurun_out; mkdir -p $OUT
for v in ${VARIANTS:-0 1 -1 0 1 -1}; do
  SS_NVCC_EXTRA="-DSS_LF_TRIGGER=$v ${EXTRA:-}" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $(timeout 600 python -m pytest tests -m gpu -q -x -k 'lastframe or ring' -p no:cacheprovider 2>&1 | tail -1)"
  for K in 200 20; do
    timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/lft.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/lft.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  [$v] K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'lastframe', round(k['lastframe'],1), 'match_window', round(k['match_window'],1), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
