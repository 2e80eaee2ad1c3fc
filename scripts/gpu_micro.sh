#!/bin/bash
# One gpurun call: integer-pipe peak microbenchmarks (scripts/micro/int_peaks.cu) under the
# clocks sampler, then (optionally) the default bench.  Usage: bash scripts/gpu_micro.sh TAG
set -u
TAG=${1:-r02}
OUT=gpurun_out
mkdir -p $OUT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o /tmp/int_peaks scripts/micro/int_peaks.cu || exit 1
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 100 > $OUT/micro_clocks_$TAG.csv &
SMI=$!
for i in 1 2 3; do /tmp/int_peaks > $OUT/int_peaks_${TAG}_$i.json; done
kill $SMI
cat $OUT/int_peaks_${TAG}_3.json
if [ "${WITH_NCU:-1}" = "1" ]; then
  ncu --metrics smsp__inst_executed_pipe_alu.sum,smsp__inst_executed_pipe_fma.sum,smsp__inst_executed_pipe_fmaheavy.sum,smsp__inst_executed_pipe_fmalite.sum,smsp__inst_executed_pipe_xu.sum,smsp__inst_executed_pipe_uniform.sum,smsp__inst_executed.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,gpu__time_duration.sum \
    --clock-control none --csv --log-file $OUT/int_peaks_ncu_$TAG.csv -c 40 /tmp/int_peaks > /dev/null 2>&1
  echo "ncu rc=$?"
fi
