#!/bin/bash
# FAST segment-size sweep (SS_SEG0 = cells per level-0 segment, SS_SEG1 = levels >= 1)
OUT=gpurun_out; mkdir -p $OUT
[ "${SKIP_TESTS:-0}" = 1 ] || timeout 600 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_seg.txt 2>&1; tail -2 $OUT/pytest_gpu_seg.txt
for s in ${SEGS:-"8 8" "12 12" "24 24" "8 16" "6 8" "10 10" "8 8"}; do
  set -- $s
  SS_SEG0=$1 SS_SEG1=$2 timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline > $OUT/seg_$1_$2.json 2>/dev/null
  python - $1 $2 <<'PY'
import json,sys
d=json.loads(open(f"gpurun_out/seg_{sys.argv[1]}_{sys.argv[2]}.json").read().strip().splitlines()[-1])
k=d["kernels_us"]
print(sys.argv[1], sys.argv[2], round(d["value"]), round(d["latency_ms"]["p50"],4), round(d["latency_ms"]["isolated_tick_ms"],4), round(k["fast_l0"],1), round(k["fast_l1plus"],1), round(d["e2e"]["value"]))
PY
done
