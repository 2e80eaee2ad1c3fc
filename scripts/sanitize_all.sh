#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over scripts/sanitize_extract.py
mkdir -p gpurun_out/sanitizer
python -c "from paper_conf_conext_dhakalrwcr22_b200 import build as b; b.build()"
for t in memcheck racecheck synccheck; do
  EX=""; [ $t = racecheck ] && EX="--kernel-name-exclude kns=brute_tc_kernel"  # see tests/test_gpu_parity.py
  timeout 900 compute-sanitizer --tool $t --error-exitcode 9 $EX python scripts/sanitize_extract.py > gpurun_out/sanitizer/san_$t.txt 2>&1
  echo "$t rc=$?"; tail -2 gpurun_out/sanitizer/san_$t.txt
done
