#!/bin/bash
# GPU box (gpurun): parity tests, ill-conditioned iteration spread, sanitizers
# on every kernel family.  usage: tools/r2_check.sh <tag>
set -u
TAG=${1:-r2}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke_$TAG.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log
timeout 600 python tools/iter_sensitivity.py --gpu --n 1000 --out $OUT/iter_sensitivity_$TAG.json \
    > $OUT/iter_sensitivity_$TAG.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $tool python tools/sanitize_cases.py (SAN_BATCH=3)" >> $OUT/sanitizer_$TAG.txt
  SAN_BATCH=3 timeout 900 compute-sanitizer --tool $tool python tools/sanitize_cases.py \
      >> $OUT/sanitizer_$TAG.txt 2>&1
  echo "rc=$?" >> $OUT/sanitizer_$TAG.txt
done
echo done
