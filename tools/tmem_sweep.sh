#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/tmem_sweep.txt
run() { timeout 300 python bench.py --steps 5 --warmup 2 --no-e2e --no-cpu-baseline "$@" 2>&1 | tail -1 | \
  python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', 'G='+__import__('os').environ.get('BSOLVE_TMEM_GROUP','2'), round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],3))" >> $OUT/tmem_sweep.txt 2>&1; }
run
for g in 1 2 4; do BSOLVE_TMEM_GROUP=$g run --placement tmem; done
