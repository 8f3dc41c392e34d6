#!/bin/bash
# generic-width line kernels: GPU tests + A/B bench vs the compile-time width (tools/r2_generic.sh <tag>)
set -u
TAG=${1:-gen}
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_blockjacobi.py -x -q > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/summary_$TAG.txt
for rep in 1 2; do
for gk in 0 1; do
  BSOLVE_LINE_GENERIC=$gk timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline \
     --parity none > $OUT/bench_${TAG}_$gk.log 2>&1
  tail -1 $OUT/bench_${TAG}_$gk.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('generic=$gk', round(d['value']/1e6,3), d['plan'].get('line_generic'), d['plan'].get('regs_per_thread'))" >> $OUT/summary_$TAG.txt 2>&1
done; done
for g in "40 25" "24 40" "100 10"; do
  set -- $g
  timeout 600 python bench.py --nx $1 --ny $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline \
     --parity none > $OUT/bench_${TAG}_$1x$2.log 2>&1
  tail -1 $OUT/bench_${TAG}_$1x$2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); s=d['solve_stats']; print('$1x$2', round(d['value']/1e6,3), 'Msys/s it', round(s['iters_mean_ion'],2), round(s['iters_mean_electron'],2), d['plan'].get('line_generic'), d['plan'].get('kernel_mode'))" >> $OUT/summary_$TAG.txt 2>&1
  BSOLVE_TMEM_LINE=0 timeout 600 python bench.py --nx $1 --ny $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline \
     --parity none > $OUT/bench_${TAG}_$1x$2_strided.log 2>&1
  tail -1 $OUT/bench_${TAG}_$1x$2_strided.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1x$2 strided', round(d['value']/1e6,3), d['plan'].get('kernel_mode'))" >> $OUT/summary_$TAG.txt 2>&1
done
cat $OUT/summary_$TAG.txt; tail -3 $OUT/pytest_$TAG.log
