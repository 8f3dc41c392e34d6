#!/bin/bash
# GPU box (gpurun): the round's closing evidence on HEAD.  usage: tools/r2_final.sh <tag>
set -u
TAG=${1:-r2f}
OUT=gpurun_out; mkdir -p $OUT
bash tools/r2_full.sh $TAG
timeout 1200 python tools/bench_configs.py --out $OUT/configs_$TAG.jsonl > $OUT/configs_$TAG.log 2>&1
echo final-done
