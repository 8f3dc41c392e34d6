#!/bin/bash
# A/B two builds of libbsolve.so on one box: tools/ab_so.sh <tag> <a.so> <b.so> [bench args]
set -u
TAG=$1; A=$2; B=$3; shift 3
OUT=gpurun_out; mkdir -p $OUT; : > $OUT/ab_$TAG.txt
LIB=paper_conf_ipps_kashinksla22_b200/libbsolve.so
for rep in 1 2 3; do
  for so in $A $B; do
    cp $so $LIB
    timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --parity none "$@" 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$so', round(d['value']/1e6,4))" >> $OUT/ab_$TAG.txt
  done
done
