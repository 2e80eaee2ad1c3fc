#!/bin/bash
# A/B of O13's frame layout: SS_LF_CLUSTER CTAs x SS_LF_THREADS threads per frame (one gpurun call).
set -u
OUT=gpurun_out; mkdir -p $OUT
# VARIANTS: comma-separated "clusters threads [lanes]" triples
IFS=, read -ra VS <<< "${VARIANTS:-1 1024,2 1024,4 512,2 512,8 512}"
for V in "${VS[@]}"; do
  set -- $V
  SS_NVCC_EXTRA="-DSS_LF_CLUSTER=$1 -DSS_LF_THREADS=$2 -DSS_LF_LANES=${3:-4}" python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  timeout 600 python -m pytest tests/test_gpu_lastframe.py -q -x -p no:cacheprovider 2>&1 | tail -1
  for C in c2 c1; do
    for rep in 1 2; do
      timeout 600 python bench.py --config $C --no-cpu-baseline > $OUT/lf_$1_$2_${C}_$rep.json 2> /dev/null
      python -c "
import json; d=json.loads(open('$OUT/lf_$1_$2_${C}_$rep.json').read().strip().splitlines()[-1])
k=d['kernels_us']; print('cl=$1 thr=$2 lanes=${3:-4} $C', round(d['value']), 'steady', round(d['steady_state']['value']), 'lastframe', round(k['lastframe'],1), 'p50', round(d['latency_ms']['p50'],4))"
    done
  done
done
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
