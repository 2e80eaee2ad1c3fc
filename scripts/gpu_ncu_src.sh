#!/bin/bash
# One gpurun call: ncu --set full with source correlation of the kernels matching a regex on
# the c2 bench (few ticks), for per-line instruction / stall analysis here.
# Usage: bash scripts/gpu_ncu_src.sh TAG 'regex' [count] [bench args...]
set -u
TAG=$1; KRX=$2; CNT=${3:-3}; shift 3 || shift $#
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$KRX" -s 30 -c $CNT -o $OUT/src_$TAG -f \
  python bench.py --steps 10 --warmup 3 --ring 8 --no-cpu-baseline "$@" > $OUT/ncu_src_$TAG.log 2>&1
echo "ncu rc=$?"; tail -3 $OUT/ncu_src_$TAG.log
