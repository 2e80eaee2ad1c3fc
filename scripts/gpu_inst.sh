#!/bin/bash
# One gpurun call: per-kernel executed instructions + device time of a few c2 ticks (ncu, cheap
# metrics only) and the multi-rank test.  Usage: bash scripts/gpu_inst.sh TAG [bench args]
set -u
TAG=$1; shift
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; exit 1; }
timeout 600 ncu --metrics smsp__inst_executed.sum,gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,launch__grid_size,launch__block_size,launch__registers_per_thread \
  --clock-control none --csv --log-file $OUT/inst_$TAG.csv -s 200 -c 120 \
  python bench.py --steps 10 --warmup 3 --ring 8 --no-cpu-baseline "$@" > $OUT/inst_$TAG.log 2>&1
echo "ncu rc=$?"
