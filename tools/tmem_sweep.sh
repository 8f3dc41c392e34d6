#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/tmem_sweep.txt
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --placement tmem 2>&1 | tail -1 | \
  python -c "import json,sys,os; d=json.loads(sys.stdin.read()); print('rounds', os.environ.get('BSOLVE_TMEM_ROUNDS'), 'G', os.environ.get('BSOLVE_TMEM_GROUP'), round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],3), 'iters', d['solve_stats']['iters_mean_electron'], d['solve_stats']['all_converged'])" >> $OUT/tmem_sweep.txt 2>&1; }
for cfg in "3 4" "2 4" "2 2"; do set -- $cfg; BSOLVE_TMEM_ROUNDS=$1 BSOLVE_TMEM_GROUP=$2 run; done
