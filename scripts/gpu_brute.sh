#!/bin/bash
# One gpurun call: build, brute-force GPU tests, three c5 benches under a watchdog.
set -u
TAG=${1:-r01}
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; }
timeout 600 python -m pytest tests/test_gpu_brute_tc.py tests/test_gpu_brute_shard.py -q -x > $OUT/pytest_brute_$TAG.txt 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_brute_$TAG.txt
for i in 1 2 3; do
  PYTHONFAULTHANDLER=1 timeout -s ABRT 300 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu-baseline \
     > $OUT/bench_${TAG}_c5_$i.json 2> $OUT/bench_${TAG}_c5_$i.err
  echo "c5 #$i rc=$?"; python -c "import json; d=json.loads(open('$OUT/bench_${TAG}_c5_$i.json').read().strip().splitlines()[-1]); print(round(d['value']), round(d['kernels_us']['brute_tc'],1), round(d['roofline']['frac'],3))" 2>&1 | tail -1
done
