#!/bin/bash
set -u
TAG=${1:-cl}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "cluster" > $OUT/pytest_$TAG.log 2>&1; BSOLVE_CLUSTER_SYNC=barrier timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "cluster" >> $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/summary_$TAG.txt
for cl in 3 3b 0; do
  SYNC=mb; [ "$cl" = "3b" ] && SYNC=barrier; BSOLVE_CLUSTER_SYNC=$SYNC BSOLVE_CLUSTER_LINE=${cl%b} timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 \
     --no-e2e --no-cpu-baseline --parity none --out $OUT/bench_${TAG}_$cl.jsonl > $OUT/bench_${TAG}_$cl.log 2>&1
  tail -1 $OUT/bench_${TAG}_$cl.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; s=d['solve_stats']; print('line=$cl', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms', 'C', p['cluster'], 'ctas', p['ctas_per_sm'], 'it', round(s['iters_mean_ion'],2), round(s['iters_mean_electron'],2), s['all_converged'])" >> $OUT/summary_$TAG.txt 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:line3_cluster -s 3 -c 1 \
    -o $OUT/prof_$TAG python bench.py --nx 64 --ny 63 --batch 16384 --steps 1 --warmup 3 --no-e2e \
    --no-cpu-baseline --parity none > $OUT/ncu_$TAG.log 2>&1
: > $OUT/racecheck_$TAG.txt
for case in "line-tiled cluster" "2-CTA cluster" "strided cluster" "cluster C=3"; do
  for sync in barrier mb; do
    echo "== racecheck case=$case BSOLVE_CLUSTER_SYNC=$sync" >> $OUT/racecheck_$TAG.txt
    BSOLVE_CLUSTER_SYNC=$sync SAN_BATCH=3 SAN_CASES="$case" timeout 600 compute-sanitizer --tool racecheck \
        python tools/sanitize_cases.py >> $OUT/racecheck_$TAG.txt 2>&1
    echo "rc=$?" >> $OUT/racecheck_$TAG.txt
  done
done
echo done
