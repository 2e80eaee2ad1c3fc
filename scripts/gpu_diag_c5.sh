#!/bin/bash
# One gpurun call: GPU tests, c2 bench, c5 bench under a watchdog (faulthandler traceback on
# SIGABRT), ncu full captures of describe (c2) and brute_tc (c5).  Usage: bash scripts/gpu_diag_c5.sh TAG
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; }
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest rc=$?" | tee -a $OUT/pytest_gpu_$TAG.txt
tail -3 $OUT/pytest_gpu_$TAG.txt
for i in 1 2; do
  PYTHONFAULTHANDLER=1 timeout -s ABRT 300 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu-baseline \
     > $OUT/bench_${TAG}_c5_$i.json 2> $OUT/bench_${TAG}_c5_$i.err
  echo "bench c5 #$i rc=$?"; tail -c 400 $OUT/bench_${TAG}_c5_$i.json; tail -30 $OUT/bench_${TAG}_c5_$i.err
done
timeout 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench c2 rc=$?"
tail -c 1500 $OUT/bench_$TAG.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:describe -s 20 -c 2 -o $OUT/prof_desc_$TAG -f \
  python bench.py --steps 10 --warmup 3 --ring 8 --no-cpu-baseline > $OUT/ncu_desc_$TAG.log 2>&1; echo "ncu desc rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:brute_tc -s 3 -c 1 -o $OUT/prof_c5_$TAG -f \
  python bench.py --config c5 --steps 4 --warmup 3 --ring 4 --inflight 1 --no-cpu-baseline > $OUT/ncu_c5_$TAG.log 2>&1; echo "ncu c5 rc=$?"
