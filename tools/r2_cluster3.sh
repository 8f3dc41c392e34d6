#!/bin/bash
set -u
TAG=${1:-cl}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "cluster" > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/summary_$TAG.txt
for sync in state halo barrier; do
  BSOLVE_CLUSTER_SYNC=$sync timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 \
     --no-e2e --no-cpu-baseline --parity none --out $OUT/bench_${TAG}_$sync.jsonl > $OUT/bench_${TAG}_$sync.log 2>&1
  tail -1 $OUT/bench_${TAG}_$sync.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; s=d['solve_stats']; print('$sync', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms', 'C', p['cluster'], 'it', round(s['iters_mean_ion'],2), round(s['iters_mean_electron'],2), s['all_converged'])" >> $OUT/summary_$TAG.txt 2>&1
done
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --parity none > $OUT/bench_${TAG}_992.log 2>&1
tail -1 $OUT/bench_${TAG}_992.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('992', round(d['value']/1e6,3))" >> $OUT/summary_$TAG.txt
for mode in 0 1 2 3; do
  timeout 300 compute-sanitizer --tool racecheck tools/cluster_race_probe $mode > $OUT/race_probe_${TAG}_$mode.txt 2>&1
  echo "rc=$?" >> $OUT/race_probe_${TAG}_$mode.txt
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:line3_cluster -s 3 -c 1 \
    -o $OUT/prof_$TAG python bench.py --nx 64 --ny 63 --batch 16384 --steps 1 --warmup 3 --no-e2e \
    --no-cpu-baseline --parity none > $OUT/ncu_$TAG.log 2>&1
echo done
