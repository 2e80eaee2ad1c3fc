#!/bin/bash
# Pyramid block-grid sweep (SS_PYR_GX x SS_PYR_GY blocks per frame) on the c2 bench.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for V in ${GRIDS:-"6 5" "6 6" "7 5" "8 5" "5 5" "8 6"}; do
  set -- $V
  SS_PYR_GX=$1 SS_PYR_GY=$2 timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k pyramid -p no:cacheprovider 2>&1 | tail -1
  for rep in 1 2; do
    SS_PYR_GX=$1 SS_PYR_GY=$2 timeout 600 python bench.py --no-cpu-baseline ${BENCH_ARGS:-} > $OUT/pyr_$1_$2_$rep.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/pyr_$1_$2_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('pyr $1x$2', round(d['value']), 'steady', round(d['steady_state']['value']), 'pyr', round(k['pyramid'],1), 'p50', round(d['latency_ms']['p50'],4))"
  done
done
