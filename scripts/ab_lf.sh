#!/bin/bash
# lastframe variants (compile-time): lanes per point / threads per CTA, c2 + c1 bench lines.
set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 300 python -m pytest tests -m gpu -q -x -k "lastframe or track" -p no:cacheprovider 2>&1 | tail -1
for V in "" "-DSS_LF_LANES=4" "-DSS_LF_LANES=2" "-DSS_LF_THREADS=512"; do
  SS_NVCC_EXTRA="$V" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  for C in c2 c1; do
    timeout 600 python bench.py --config $C --no-cpu-baseline > $OUT/lf_ab.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/lf_ab.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('[$V] $C', round(d['value']), 'steady', round(d['steady_state']['value']), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'lastframe', round(k['lastframe'],1))"
  done
done
