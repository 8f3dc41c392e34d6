#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; TAG=${1:-sweep}
run() { timeout 300 python bench.py --steps 5 --warmup 2 --no-e2e --no-cpu-baseline "$@" 2>&1 | tail -1 | \
  python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],3))" >> $OUT/$TAG.txt 2>&1; }
: > $OUT/$TAG.txt
run --placement regs
run --block-threads 128 --reg-slots 4
