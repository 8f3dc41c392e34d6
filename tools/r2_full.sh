#!/bin/bash
# GPU box (gpurun): the round's evidence in one call.  usage: tools/r2_full.sh <tag>
set -u
TAG=${1:-r2}
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke_$TAG.log 2>&1
echo "smoke rc=$?" >> $OUT/smoke_$TAG.log
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log
timeout 900 python bench.py --steps 10 --warmup 3 --out $OUT/bench_$TAG.jsonl > $OUT/bench_$TAG.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $OUT/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --cpu-seconds 2 \
    --parity sample > $OUT/ncu_launch_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bicgstab -s 3 -c 1 \
    -o $OUT/prof_$TAG python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --parity none \
    > $OUT/ncu_full_$TAG.log 2>&1
timeout 900 python bench.py --picard 5 --steps 3 --warmup 1 --out $OUT/picard_$TAG.jsonl > $OUT/picard_$TAG.log 2>&1
timeout 600 python tools/iter_sensitivity.py --gpu --n 1000 --out $OUT/iter_sensitivity_$TAG.json \
    > $OUT/iter_sensitivity_$TAG.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $tool python tools/sanitize_cases.py (SAN_BATCH=3, line-tiled cases)" >> $OUT/sanitizer_$TAG.txt
  SAN_BATCH=3 SAN_CASES=line-tiled timeout 900 compute-sanitizer --tool $tool python tools/sanitize_cases.py \
      >> $OUT/sanitizer_$TAG.txt 2>&1
  echo "rc=$?" >> $OUT/sanitizer_$TAG.txt
done
timeout 300 compute-sanitizer --tool synccheck tools/tmem_probe > $OUT/synccheck_tmem_probe_$TAG.txt 2>&1
echo "rc=$?" >> $OUT/synccheck_tmem_probe_$TAG.txt
echo done
