#!/bin/bash
# One gpurun call: build, GPU tests, default (c2) bench, ncu full capture of one kernel.
# Usage: bash scripts/gpu_quick.sh TAG [kernel-regex] [extra bench configs...]
set -u
TAG=${1:-r01}; KRX=${2:-describe}; shift 2 || true
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; }
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest rc=$?" | tee -a $OUT/pytest_gpu_$TAG.txt
tail -3 $OUT/pytest_gpu_$TAG.txt
timeout 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench c2 rc=$?"
for C in "$@"; do
  PYTHONFAULTHANDLER=1 timeout -s ABRT 400 python bench.py --config $C --steps 50 --warmup 5 --no-cpu-baseline \
     > $OUT/bench_${TAG}_$C.json 2> $OUT/bench_${TAG}_$C.err; echo "bench $C rc=$?"; tail -20 $OUT/bench_${TAG}_$C.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$KRX" -s 20 -c 2 -o $OUT/prof_k_$TAG -f \
  python bench.py --steps 10 --warmup 3 --ring 8 --no-cpu-baseline > $OUT/ncu_k_$TAG.log 2>&1; echo "ncu rc=$?"
