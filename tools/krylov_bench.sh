#!/bin/bash
# Run on the GPU box: bench.py lines for the f3 solvers (GMRES(m), no preconditioner).
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/krylov_bench.jsonl
for a in "--solver gmres --restart 7" "--solver gmres --restart 4" "--precond none" "--solver gmres --precond none"; do
  timeout 400 python bench.py --steps 5 --warmup 3 --no-e2e --cpu-seconds 5 $a 2>&1 | tail -1 >> $OUT/krylov_bench.jsonl
done
