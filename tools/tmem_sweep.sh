#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/tmem_sweep.txt
run() { timeout 300 python bench.py --steps 5 --warmup 2 --no-e2e --no-cpu-baseline --placement tmem 2>&1 | tail -1 | \
  python -c "import json,sys,os; d=json.loads(sys.stdin.read()); print('threads', os.environ.get('BSOLVE_TMEM_THREADS'), 'G', os.environ.get('BSOLVE_TMEM_GROUP'), round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],3), 'ctas/sm', d['plan']['ctas_per_sm'])" >> $OUT/tmem_sweep.txt 2>&1; }
for cfg in "128 4" "256 1" "256 2"; do set -- $cfg; BSOLVE_TMEM_THREADS=$1 BSOLVE_TMEM_GROUP=$2 run; done
