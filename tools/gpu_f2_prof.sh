#!/bin/bash
# GPU box: ncu --set full of the n = 4032 cluster kernel.  usage: tools/gpu_f2_prof.sh <tag>  (env passes through)
set -u
TAG=${1:-f2}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cluster -s 1 -c 1 \
    -o $OUT/f2_prof_$TAG python bench.py --nx 64 --ny 63 --batch 4096 --steps 1 --warmup 1 --no-e2e \
    --no-cpu-baseline --parity none > $OUT/f2_ncu_full_$TAG.log 2>&1
echo done
