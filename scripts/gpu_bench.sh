#!/bin/bash
# One gpurun call: GPU parity tests, default bench, ncu launch list + a full capture of the top kernels.
# Usage (from the repo root, on the GPU box): bash scripts/gpu_bench.sh [tag]
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/smi_$TAG.txt 2>&1
if [ "${SKIP_TESTS:-0}" != "1" ]; then
  timeout 900 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.txt
  tail -3 $OUT/pytest_gpu_$TAG.txt
fi
timeout 300 python __graft_entry__.py smoke > $OUT/smoke_$TAG.txt 2>&1; echo "smoke rc=$?"; tail -2 $OUT/smoke_$TAG.txt
timeout 900 python bench.py ${BENCH_ARGS:-} > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err; echo "bench rc=$?"
tail -c 3000 $OUT/bench_$TAG.json
tail -5 $OUT/bench_$TAG.err
for C in ${EXTRA_CONFIGS:-}; do
  PYTHONFAULTHANDLER=1 timeout -s ABRT 600 python bench.py --config $C --steps 50 --warmup 5 --no-cpu-baseline > $OUT/bench_${TAG}_$C.json 2> $OUT/bench_${TAG}_$C.err
  echo "bench $C rc=$?"; tail -c 600 $OUT/bench_${TAG}_$C.json
done
if [ "${SKIP_NCU:-0}" != "1" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv \
     python bench.py --steps 20 --warmup 3 --ring 8 --no-cpu-baseline ${NCU_BENCH_ARGS:-} > $OUT/ncu_bench_$TAG.log 2>&1
  echo "ncu list rc=$?"
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"${NCU_KERNELS:-fast_bands|distribute|describe|match_window|pyramid|project|match_prepare|match_window_resolve|lastframe}" \
     -s ${NCU_SKIP:-40} -c ${NCU_COUNT:-12} -o $OUT/prof_$TAG -f \
     python bench.py --steps 20 --warmup 3 --ring 8 --no-cpu-baseline ${NCU_BENCH_ARGS:-} > $OUT/ncu_full_$TAG.log 2>&1
  echo "ncu full rc=$?"
fi
