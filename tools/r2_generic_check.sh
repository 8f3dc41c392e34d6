#!/bin/bash
# generic-width line kernels: all GPU tests + sanitizers on the generic cases (tools/r2_generic_check.sh <tag>)
set -u
TAG=${1:-genc}
OUT=gpurun_out; mkdir -p $OUT
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log
: > $OUT/sanitizer_$TAG.txt
for tool in memcheck racecheck initcheck; do
  echo "== compute-sanitizer --tool $tool (SAN_CASES=generic,bench default)" >> $OUT/sanitizer_$TAG.txt
  SAN_BATCH=3 SAN_CASES="generic,bench default" timeout 900 compute-sanitizer --tool $tool \
      python tools/sanitize_cases.py >> $OUT/sanitizer_$TAG.txt 2>&1
  echo "rc=$?" >> $OUT/sanitizer_$TAG.txt
done
tail -3 $OUT/pytest_gpu_$TAG.log; grep -E "^==|SUMMARY|ok$|FAIL" $OUT/sanitizer_$TAG.txt
