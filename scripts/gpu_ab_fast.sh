#!/bin/bash
# A/B of the FAST kernel's CTA shape (SS_FAST_WARPS, SS_FAST_ROWS) on the c2 bench (one gpurun call).
set -u
OUT=gpurun_out; mkdir -p $OUT
for V in ${VARIANTS:-"8 8" "8 4" "16 4" "16 8" "12 8"}; do
  set -- $V
  SS_NVCC_EXTRA="-DSS_FAST_WARPS=$1 -DSS_FAST_ROWS=$2" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > $OUT/build_fast_$1_$2.txt 2>&1 || { echo build $V failed; continue; }
  timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "extract or fast" -p no:cacheprovider 2>&1 | tail -1
  for rep in 1 2; do
    timeout 600 python bench.py --no-cpu-baseline > $OUT/bench_fast_$1_$2_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/bench_fast_$1_$2_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('W=$1 R=$2', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', round(k['fast_l0'],1), round(k['fast_l1plus'],1), [r['frac'] for r in d['rooflines'] if r['kernel'].startswith('fast')])"
  done
done
