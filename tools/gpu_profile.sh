#!/bin/bash
# Run on the GPU box (via gpurun): bench line, ncu launch list of the same
# bench command, and one full ncu capture of the solve kernel.
# usage: tools/gpu_profile.sh <tag>
set -u
TAG=${1:-r1}
OUT=gpurun_out
mkdir -p $OUT
timeout 600 python bench.py --steps 10 --warmup 3 --out $OUT/bench_$TAG.jsonl > $OUT/bench_$TAG.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $OUT/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --cpu-seconds 2 \
    > $OUT/ncu_launch_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bicgstab -s 3 -c 1 \
    -o $OUT/prof_$TAG python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline \
    > $OUT/ncu_full_$TAG.log 2>&1
echo done
