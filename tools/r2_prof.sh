#!/bin/bash
# usage: tools/r2_prof.sh <tag> <kernel regex> <bench args...>   (env passes through)
set -u
TAG=$1; KR=$2; shift 2
OUT=gpurun_out; mkdir -p $OUT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$KR -s 3 -c 1 \
    -o $OUT/prof_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --parity none "$@" \
    > $OUT/ncu_$TAG.log 2>&1
echo done
