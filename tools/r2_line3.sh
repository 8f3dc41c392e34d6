#!/bin/bash
# GPU box: 3-CTA line kernel (line3_kernel.cuh) vs the 2-CTA line kernel:
# parity tests under each plan, bench lines, one ncu capture.
set -u
TAG=${1:-l3}
OUT=gpurun_out; mkdir -p $OUT
run() { local tag=$1; shift; env "$@" timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e \
  --no-cpu-baseline --out $OUT/bench_${TAG}_$tag.jsonl > $OUT/bench_${TAG}_$tag.log 2>&1;
  tail -1 $OUT/bench_${TAG}_$tag.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; s=d['solve_stats']; print('$tag', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],3), 'regs', p.get('regs_per_thread'), 'ctas', p['ctas_per_sm'], 'it', round(s['iters_mean_ion'],3), round(s['iters_mean_electron'],3), 'conv', s['all_converged'], 'clk', d['clocks'].get('sm_mhz'))" >> $OUT/summary_$TAG.txt 2>&1; }
: > $OUT/summary_$TAG.txt
for cfg in "BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=2 BSOLVE_LINE3_GROUP=3"; do
  env $cfg timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q \
     > "$OUT/pytest_${TAG}_${cfg// /_}.log" 2>&1; echo "pytest $cfg rc=$?" >> $OUT/summary_$TAG.txt
done
run base BSOLVE_LINE_CTAS=2
run c3g3r3 BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=3 BSOLVE_LINE3_GROUP=3
run c3g3r2 BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=2 BSOLVE_LINE3_GROUP=3
run c3r3 BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=3
run c3r2 BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=2

timeout 600 ncu --set full --clock-control none --import-source on -k regex:line3 -s 3 -c 1 \
    -o $OUT/prof_${TAG}_c3g3r2 env BSOLVE_LINE_CTAS=3 BSOLVE_ROUNDS=2 BSOLVE_LINE3_GROUP=3 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
    > $OUT/ncu_${TAG}_c3r2.log 2>&1
echo done
