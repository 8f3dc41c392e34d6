#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/tmem_persist_sweep.txt
for pp in 1 0; do
  BSOLVE_TMEM_PERSIST=$pp timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | \
  python -c "import json,sys; d=json.loads(sys.stdin.read()); print('persist=$pp', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],3))" >> $OUT/tmem_persist_sweep.txt
done
