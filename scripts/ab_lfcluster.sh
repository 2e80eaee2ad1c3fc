#!/bin/bash
# lastframe CTAs per frame (compile-time SS_LF_CLUSTER): parity tests + c2 / c1 bench lines.
set -u
OUT=gpurun_out; mkdir -p $OUT
for C in 2 4 1; do
  SS_NVCC_EXTRA="-DSS_LF_CLUSTER=$C" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "cluster=$C: $(timeout 300 python -m pytest tests -m gpu -q -x -k 'lastframe or track' -p no:cacheprovider 2>&1 | tail -1)"
  for C2 in c2 c1; do
    for K in 200 20; do
      timeout 600 python bench.py --config $C2 --steps $K --warmup 5 --no-cpu-baseline > $OUT/lfc.json 2> /dev/null
      python -c "
import json; d=json.loads(open('$OUT/lfc.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('  cluster=$C $C2 K=$K', round(d['value']), 'steady', round((d.get('steady_state') or {}).get('value') or 0), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'lastframe', round(k['lastframe'],1))"
    done
  done
done
