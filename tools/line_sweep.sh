#!/bin/bash
# Run on the GPU box: bench.py of the line-tiled TMEM kernel for each geometry
# (rows per thread x TMEM load group), and of the strided TMEM kernels
# (BSOLVE_TMEM_LINE=0) for reference.
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/line_sweep.txt
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | \
  python -c "import json,sys,os; d=json.loads(sys.stdin.read()); e=os.environ.get; print('line', e('BSOLVE_TMEM_LINE'), 'rows', e('BSOLVE_TMEM_LINE_ROWS'), 'G', e('BSOLVE_TMEM_GROUP'), 'thr', e('BSOLVE_TMEM_THREADS'), 'mode', d['plan']['kernel_mode'], 'R', d['plan']['rows_per_thread'], round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],3), 'iters', d['solve_stats']['iters_mean_electron'], d['solve_stats']['all_converged'])" >> $OUT/line_sweep.txt 2>&1; }
for cfg in "8 4" "8 2" "4 2"; do set -- $cfg; BSOLVE_TMEM_LINE_ROWS=$1 BSOLVE_TMEM_GROUP=$2 run; done
BSOLVE_TMEM_LINE=0 run
BSOLVE_TMEM_LINE=0 BSOLVE_TMEM_THREADS=256 run
