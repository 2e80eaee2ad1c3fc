#!/bin/bash
# pyramid block grid (SS_PYR_GX x SS_PYR_GY per frame) on c3 (16 TUM frames) and c2.
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for C in c3 c2; do
  for V in "0 0" "3 3" "4 4" "4 3" "6 5" "8 6"; do
    set -- $V
    if [ $1 = 0 ]; then unset SS_PYR_GX SS_PYR_GY; else export SS_PYR_GX=$1 SS_PYR_GY=$2; fi
    timeout 600 python bench.py --config $C --steps 100 --warmup 5 --no-cpu-baseline > $OUT/pyr.json 2> /dev/null
    python -c "
import json; d=json.loads(open('$OUT/pyr.json').read().strip().splitlines()[-1])
k=d['kernels_us']; r=[x for x in d['rooflines'] if x['kernel']=='pyramid'][0]
print('$C grid=$1x$2', round(d['value']), 'pyramid', round(k['pyramid'],1), 'hbm frac', round(r['frac'],3))"
  done
done
