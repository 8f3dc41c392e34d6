#!/bin/bash
# A/B of the cluster exchange variants (f2): tools/r2_state.sh
set -u
OUT=gpurun_out; mkdir -p $OUT; TAG=st1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "cluster" > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/summary_$TAG.txt
for rep in 1 2; do
for sync in state halo; do
  BSOLVE_CLUSTER_SYNC=$sync timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 \
     --no-e2e --no-cpu-baseline --parity none > $OUT/bench_${TAG}_$sync.log 2>&1
  tail -1 $OUT/bench_${TAG}_$sync.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; s=d['solve_stats']; print('$sync', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms', 'C', p['cluster'], 'it', round(s['iters_mean_ion'],2), round(s['iters_mean_electron'],2), s['all_converged'])" >> $OUT/summary_$TAG.txt 2>&1
done; done
for ny in 31 95 127; do
for sync in state halo; do
  BSOLVE_CLUSTER_SYNC=$sync timeout 600 python bench.py --nx 64 --ny $ny --batch 8192 --steps 10 --warmup 3 \
     --no-e2e --no-cpu-baseline --parity none > $OUT/bench_${TAG}_$sync.log 2>&1
  tail -1 $OUT/bench_${TAG}_$sync.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; print('ny$ny $sync', round(d['value']/1e6,3), p['cluster'])" >> $OUT/summary_$TAG.txt 2>&1
done; done
cat $OUT/summary_$TAG.txt; tail -3 $OUT/pytest_$TAG.log
