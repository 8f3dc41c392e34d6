#!/bin/bash
# Run on the GPU box: bench line of the f4 banded direct solver, the ncu launch
# list of the same command, and one full ncu capture of the banded kernel.
# usage: tools/f4_profile.sh <tag>
set -u
TAG=${1:-r1}
OUT=gpurun_out
mkdir -p $OUT
timeout 600 python bench.py --solver banded --steps 5 --warmup 3 --cpu-seconds 5 \
    --out $OUT/f4_bench_$TAG.jsonl > $OUT/f4_bench_$TAG.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $OUT/f4_launches_$TAG.csv python bench.py --solver banded --steps 3 --warmup 3 \
    --no-e2e --no-cpu-baseline > $OUT/f4_ncu_launch_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:banded_lu -s 3 -c 1 \
    -o $OUT/f4_prof_$TAG python bench.py --solver banded --steps 1 --warmup 3 --no-e2e \
    --no-cpu-baseline > $OUT/f4_ncu_full_$TAG.log 2>&1
echo done
