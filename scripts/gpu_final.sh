#!/bin/bash
# The round's evidence in one gpurun call: GPU tests, smoke, every config's bench line, the
# reference arm, the ncu launch list of the default bench and one `--set full` capture of its
# kernels (summary + per-launch DRAM traffic for bench.py's roofline.traffic).
# Usage: bash scripts/gpu_final.sh TAG
set -u
TAG=${1:-r02}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; exit 1; }
if [ "${SKIP_TESTS:-0}" != "1" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest rc=$?" | tee -a $OUT/pytest_gpu_$TAG.txt
  tail -3 $OUT/pytest_gpu_$TAG.txt
  timeout 300 python __graft_entry__.py smoke > $OUT/smoke_$TAG.txt 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke_$TAG.txt
fi
timeout 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench c2 rc=$?"
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > $OUT/bench_${TAG}_k20.json 2> /dev/null; echo "bench c2 K=20 rc=$?"
for C in c1 c3 c4 c5; do
  PYTHONFAULTHANDLER=1 timeout -s ABRT 600 python bench.py --config $C --no-cpu-baseline > $OUT/bench_${TAG}_$C.json 2> $OUT/bench_${TAG}_$C.err
  echo "bench $C rc=$?"
done
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_${TAG}_reference.json 2> /dev/null; echo "reference rc=$?"
python - $OUT $TAG <<'PY'
import json, sys
out, tag = sys.argv[1], sys.argv[2]
for suf in ("", "_k20", "_c1", "_c3", "_c4", "_c5", "_reference"):
    try:
        d = json.loads(open(f"{out}/bench_{tag}{suf}.json").read().strip().splitlines()[-1])
        r = d.get("roofline") or {}
        print(suf or "_c2", round(d["value"]), "e2e", round((d.get("e2e") or {}).get("value") or 0),
              "steady", round((d.get("steady_state") or {}).get("value") or 0),
              "p50", round((d.get("latency_ms") or {}).get("p50", 0), 4), r.get("kernel"), round(r.get("frac", 0), 4))
    except Exception as e:
        print(suf, "parse failed", e)
PY
if [ "${SKIP_NCU:-0}" != "1" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 400 --csv --log-file $OUT/launches_$TAG.csv \
     python bench.py --steps 20 --warmup 3 --ring 8 --no-cpu-baseline > $OUT/ncu_list_$TAG.log 2>&1
  echo "ncu list rc=$?"
  timeout 1500 ncu --set full --clock-control none --import-source on \
     -k regex:"fast_bands|distribute|describe|match_window|pyramid|project|lastframe" -s 60 -c 22 -o $OUT/full_$TAG -f \
     python bench.py --steps 20 --warmup 3 --ring 8 --no-cpu-baseline > $OUT/ncu_full_$TAG.log 2>&1
  echo "ncu full rc=$?"
fi
