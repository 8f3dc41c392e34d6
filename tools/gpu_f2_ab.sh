#!/bin/bash
# GPU box: n = 4032 cluster plan A/B over developer knobs.  usage: tools/gpu_f2_ab.sh <tag> "<ENV=..>" ...
set -u
TAG=$1; shift
OUT=gpurun_out; mkdir -p $OUT
i=0
for envs in "$@"; do
  env $envs timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
    --parity none --out $OUT/f2_${TAG}_$i.jsonl > $OUT/f2_${TAG}_$i.log 2>&1
  echo "$i: $envs" >> $OUT/f2_${TAG}_index.txt
  i=$((i+1))
done
echo done
