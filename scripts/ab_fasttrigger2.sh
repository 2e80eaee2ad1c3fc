#!/bin/bash
# Where FAST's PDL trigger sits (SS_FAST_TRIGGER: 0 = CTA start, 2 = after its scores, 3 = after
# its NMS): the distribution's CTAs (215 KB shared memory each) sit resident from then on.
set -u
OUT=gpurun_out; mkdir -p $OUT
for v in ${VARIANTS:-0 2 3 0 2 3}; do
  SS_NVCC_EXTRA="-DSS_FAST_TRIGGER=$v ${EXTRA:-}" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $(timeout 600 python -m pytest tests -m gpu -q -x -k 'parity and extract' -p no:cacheprovider 2>&1 | tail -1)"
  for K in 200 20; do
    timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/fst.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/fst.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  [$v] K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', round(k['fast'],1), 'distribute', round(k['distribute'],1), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
