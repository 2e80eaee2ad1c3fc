#!/bin/bash
# One gpurun call: build, GPU tests, distribution phase timeline, c2 bench (+ extra configs).
# Usage: bash scripts/gpu_dist.sh TAG [configs...]
set -u
TAG=${1:-d}; shift || true
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.txt 2>&1 || { echo build failed; tail -20 $OUT/build_$TAG.txt; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu_$TAG.txt
timeout 120 python scripts/diag_phases.py > $OUT/phases_$TAG.txt 2>&1; cat $OUT/phases_$TAG.txt | cut -c1-250
BENCH_ARGS="${BENCH_ARGS:-}" SKIP_TESTS=1 bash scripts/gpu_round.sh $TAG "$@" 2>&1 | grep -v "^pytest\|^smoke"
