#!/bin/bash
set -u
TAG=${1:-cl}
OUT=gpurun_out; mkdir -p $OUT
BSOLVE_CLUSTER_SYNC=barrier timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "cluster" > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/racecheck_$TAG.txt
for sync in barrier mb; do
  echo "== racecheck line3 cluster BSOLVE_CLUSTER_SYNC=$sync" >> $OUT/racecheck_$TAG.txt
  BSOLVE_CLUSTER_SYNC=$sync SAN_BATCH=3 SAN_CASES="line-tiled cluster" timeout 600 compute-sanitizer --tool racecheck \
      python tools/sanitize_cases.py >> $OUT/racecheck_$TAG.txt 2>&1
  echo "rc=$?" >> $OUT/racecheck_$TAG.txt
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:line3_cluster -s 3 -c 1 \
    -o $OUT/prof_$TAG python bench.py --nx 64 --ny 63 --batch 16384 --steps 1 --warmup 3 --no-e2e \
    --no-cpu-baseline --parity none > $OUT/ncu_$TAG.log 2>&1
echo done
