#!/bin/bash
# f4 one-warp-per-system factorisation: banded GPU tests + A/B bench (tools/r2_f4warp.sh <tag>)
set -u
TAG=${1:-f4w}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_banded.py -x -q > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/summary_$TAG.txt
for rep in 1 2; do
for wk in 1 0; do
  BSOLVE_BANDED_WARP=$wk timeout 600 python bench.py --solver banded --steps 5 --warmup 3 \
     --no-e2e --no-cpu-baseline > $OUT/bench_${TAG}_$wk.log 2>&1
  tail -1 $OUT/bench_${TAG}_$wk.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('warp=$wk', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms frac', r.get('frac'))" >> $OUT/summary_$TAG.txt 2>&1
done; done
cat $OUT/summary_$TAG.txt; tail -3 $OUT/pytest_$TAG.log
