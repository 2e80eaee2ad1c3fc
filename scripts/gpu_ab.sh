#!/bin/bash
# A/B of two prebuilt libss.so variants (gpurun_alt_*.bin at the repo root) on the c2 bench,
# interleaved A B A B on one box; then a ticks-in-flight sweep with the last variant.
set -u
TAG=${1:-ab}; shift
OUT=gpurun_out; mkdir -p $OUT
LIB=paper_conf_conext_dhakalrwcr22_b200/libss.so
for rep in 1 2; do for V in "$@"; do
  cp gpurun_alt_$V.bin $LIB
  timeout 600 python bench.py --no-cpu-baseline > $OUT/ab_${TAG}_${V}_$rep.json 2>/dev/null
  python -c "import json,sys; d=json.loads(open('$OUT/ab_${TAG}_${V}_$rep.json').read().strip().splitlines()[-1]); print('$V', $rep, round(d['value']), round(d['kernels_us']['describe'],2), round(d['e2e']['value']))"
done; done
for P in ${SWEEP:-}; do
  timeout 600 python bench.py --no-cpu-baseline --inflight $P > $OUT/ab_${TAG}_inflight$P.json 2>/dev/null
  python -c "import json; d=json.loads(open('$OUT/ab_${TAG}_inflight$P.json').read().strip().splitlines()[-1]); print('inflight $P', round(d['value']), d['latency_ms']['p50'])"
done
