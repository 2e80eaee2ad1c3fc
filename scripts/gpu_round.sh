#!/bin/bash
# One gpurun call: build, GPU tests, smoke, default (c2) bench, optional extra configs.
# Usage: bash scripts/gpu_round.sh TAG [extra configs...]   (env SKIP_TESTS=1, BENCH_ARGS=...)
set -u
TAG=${1:-r02}; shift || true
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; exit 1; }
if [ "${SKIP_TESTS:-0}" != "1" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest rc=$?" | tee -a $OUT/pytest_gpu_$TAG.txt
  tail -4 $OUT/pytest_gpu_$TAG.txt
  timeout 300 python __graft_entry__.py smoke > $OUT/smoke_$TAG.txt 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke_$TAG.txt
fi
PYTHONFAULTHANDLER=1 timeout -s ABRT 900 python bench.py ${BENCH_ARGS:-} > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench c2 rc=$?"
python - $OUT/bench_$TAG.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print("c2", round(d["value"]), "e2e", round(d["e2e"]["value"] or 0), "steady", round((d.get("steady_state") or {}).get("value", 0)),
          "p50", round(d["latency_ms"]["p50"], 4), "iso", round(d["latency_ms"]["isolated_tick_ms"], 4), d["roofline"]["kernel"], round(d["roofline"]["frac"], 3))
    print({k: round(v, 1) for k, v in sorted(d["kernels_us"].items(), key=lambda x: -x[1])})
except Exception as e:
    print("parse failed", e)
PY
for C in "$@"; do
  PYTHONFAULTHANDLER=1 timeout -s ABRT 500 python bench.py --config $C --steps 100 --warmup 5 --no-cpu-baseline ${BENCH_ARGS:-} \
     > $OUT/bench_${TAG}_$C.json 2> $OUT/bench_${TAG}_$C.err; echo "bench $C rc=$?"
  python - $OUT/bench_${TAG}_$C.json $C <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[2], round(d["value"]), "e2e", round(d["e2e"]["value"] or 0), "iso", round(d["latency_ms"]["isolated_tick_ms"], 4), d["roofline"]["kernel"], round(d["roofline"]["frac"], 3))
    print({k: round(v, 1) for k, v in sorted(d["kernels_us"].items(), key=lambda x: -x[1])})
except Exception as e:
    print("parse failed", e)
PY
done
