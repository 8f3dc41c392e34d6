#!/bin/bash
set -u
TAG=${1:-l3}
OUT=gpurun_out; mkdir -p $OUT
run() { local tag=$1; shift; env "$@" timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e \
  --no-cpu-baseline --out $OUT/bench_${TAG}_$tag.jsonl > $OUT/bench_${TAG}_$tag.log 2>&1;
  tail -1 $OUT/bench_${TAG}_$tag.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; s=d['solve_stats']; print('$tag', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],3), 'regs', p.get('regs_per_thread'), 'ctas', p['ctas_per_sm'], 'it', round(s['iters_mean_ion'],3), round(s['iters_mean_electron'],3), 'conv', s['all_converged'], 'clk', d['clocks'].get('sm_mhz'))" >> $OUT/summary_$TAG.txt 2>&1; }
: > $OUT/summary_$TAG.txt
C="BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=2"
for rep in 1 2; do
run g3_$rep $C BSOLVE_LINE3_GROUP=3
run g4_$rep $C BSOLVE_LINE3_GROUP=4
run g5_$rep $C BSOLVE_LINE3_GROUP=5
done
echo done
