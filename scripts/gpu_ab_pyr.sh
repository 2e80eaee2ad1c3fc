#!/bin/bash
# A/B of the pyramid CTA size (SS_PYR_THREADS) on the c2 bench: one gpurun call.
set -u
OUT=gpurun_out; mkdir -p $OUT
for PT in ${PTS:-1024 512 256}; do
  SS_NVCC_EXTRA="-DSS_PYR_THREADS=$PT" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > $OUT/build_pt$PT.txt 2>&1 || { echo build $PT failed; tail $OUT/build_pt$PT.txt; continue; }
  if [ "${TESTS:-0}" = "1" ]; then timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k pyramid -p no:cacheprovider 2>&1 | tail -1; fi
  for rep in 1 2; do
    timeout 600 python bench.py --no-cpu-baseline > $OUT/bench_pt${PT}_$rep.json 2> $OUT/bench_pt${PT}_$rep.err
    python -c "
import json; d=json.loads(open('$OUT/bench_pt${PT}_$rep.json').read().strip().splitlines()[-1])
print('PT=$PT', round(d['value']), 'steady', round(d['steady_state']['value']), 'iso', round(d['latency_ms']['isolated_tick_ms'],4), 'p50', round(d['latency_ms']['p50'],4), 'pyr', round(d['kernels_us']['pyramid'],1))"
  done
done
