#!/bin/bash
# describe warps (keypoints) per CTA: SS_DESC_WARPS = 8 (default) / 4 / 6, c2 (+ parity tests for each).
set -u
OUT=gpurun_out; mkdir -p $OUT
for Wp in 4 6 8; do
  SS_NVCC_EXTRA="-DSS_DESC_WARPS=$Wp" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "warps=$Wp: $(timeout 600 python -m pytest tests -m gpu -q -x -k 'parity or coverage' -p no:cacheprovider 2>&1 | tail -1)"
  for rep in 1 2; do
    timeout 600 python bench.py --no-cpu-baseline > $OUT/dw.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/dw.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  warps=$Wp', round(d['value']), 'steady', round(d['steady_state']['value']), 'describe', round(k['describe'],1), 'iso', round(d['latency_ms']['isolated_tick_ms'],4))"
  done
done
