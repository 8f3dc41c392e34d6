#!/bin/bash
# GPU box: one ncu --set full capture of the banded factor kernel.  usage: tools/gpu_f4_prof.sh <tag> [env...]
set -u
TAG=${1:-f4}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:banded_lu -s 1 -c 1 \
    -o $OUT/f4_prof_$TAG python bench.py --solver banded --batch 20000 --steps 1 --warmup 1 --no-e2e \
    --no-cpu-baseline --parity none > $OUT/f4_ncu_full_$TAG.log 2>&1
echo done
