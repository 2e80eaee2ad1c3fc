#!/bin/bash
# Where the distribution's PDL trigger sits (SS_DIST_TRIGGER: 0 = after its dependency wait,
# -1 = at exit, k = after dense-path phase k).  Its dependent, describe, is ~1000 CTAs that sit
# resident (29 KB of shared memory each) from the trigger until the distribution completes.
# (An earlier run of this script also measured FAST's and describe's triggers at exit: worse.)
set -u
OUT=gpurun_out; mkdir -p $OUT
for v in ${VARIANTS:-0 -1 6 7 8 0 -1 7}; do
  X="-DSS_DIST_TRIGGER=$v"
  SS_NVCC_EXTRA="$X" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $(timeout 600 python -m pytest tests -m gpu -q -x -k 'parity and extract' -p no:cacheprovider 2>&1 | tail -1)"
  for K in 200 20; do
    timeout 600 python bench.py --steps $K --warmup 5 --no-cpu-baseline > $OUT/lt.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/lt.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  [$v] K=$K', round(d['value']), 'steady', round(d['steady_state']['value']), 'distribute', round(k['distribute'],1), 'describe', round(k['describe'],1), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
