#!/bin/bash
# Where the pyramid's PDL trigger sits (SS_PYR_TRIGGER: 0 = its start, k = once levels < k are
# built, 9 = exit): FAST launches at the trigger; its level-0 CTAs work beside the pyramid, its
# other CTAs sit resident (80 registers x 256 threads each) until the pyramid completes.
set -u
OUT=gpurun_out; mkdir -p $OUT
for v in ${VARIANTS:-0 3 5 9 0 3}; do
  SS_NVCC_EXTRA="-DSS_PYR_TRIGGER=$v ${EXTRA:-}" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $(timeout 600 python -m pytest tests -m gpu -q -x -k 'parity and extract' -p no:cacheprovider 2>&1 | tail -1)"
  for K in 200 20; do
    timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/pt.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/pt.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  [$v] K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'pyramid', round(k['pyramid'],1), 'fast', round(k['fast'],1), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
