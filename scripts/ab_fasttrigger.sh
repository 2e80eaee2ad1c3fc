#!/bin/bash
# FAST's PDL trigger at the start of every CTA (default: the distribution grid launches as soon as
# FAST's last CTA has started, and its CTAs -- 215 KB of shared memory each -- wait on SMs FAST
# has left) vs none (SS_FAST_LATE_TRIGGER: the distribution launches as FAST's CTAs exit).
set -u
OUT=gpurun_out; mkdir -p $OUT
for v in base late base late; do
  X=""; [ $v = late ] && X="-DSS_FAST_LATE_TRIGGER"
  SS_NVCC_EXTRA="$X" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $(timeout 600 python -m pytest tests -m gpu -q -x -k 'parity and extract' -p no:cacheprovider 2>&1 | tail -1)"
  for K in 200 20; do
    timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/ft.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/ft.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  [$v] K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', round(k['fast'],1), 'distribute', round(k['distribute'],1), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
