#!/bin/bash
# FAST CTA size (compile-time SS_FAST_WARPS) x segment cells (SS_SEG0 / SS_SEG), c2 bench.
set -u
OUT=gpurun_out; mkdir -p $OUT
for V in "8 8 8" "4 4 4" "4 6 6" "4 8 8"; do
  set -- $V
  SS_NVCC_EXTRA="-DSS_FAST_WARPS=$1" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  for rep in 1 2; do
    SS_SEG0=$2 SS_SEG=$3 timeout 600 python bench.py --no-cpu-baseline > $OUT/fw_$1_$2_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/fw_$1_$2_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('warps=$1 seg=$2/$3', round(d['value']), 'steady', round(d['steady_state']['value']), 'fast', round(k['fast'],1), 'frac', round(d['roofline']['frac'],3), 'iso', round(d['latency_ms']['isolated_tick_ms'],4))"
  done
done
