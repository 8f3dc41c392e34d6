#!/bin/bash
# GPU box: default-workload bench A/B over env settings, 2 reps each.  usage: tools/gpu_env_ab.sh <tag> "<ENV=..>" ...
set -u
TAG=$1; shift
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/envab_$TAG.txt
for rep in 1 2; do
  for envs in "$@"; do
    env $envs timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --parity none 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$envs', round(d['value']/1e6,4))" >> $OUT/envab_$TAG.txt
  done
done
echo done
