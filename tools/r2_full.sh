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
timeout 600 python bench.py --precond block_jacobi --steps 10 --warmup 3 --no-e2e --parity sample --cpu-seconds 3 \
    --out $OUT/bench_bj_$TAG.jsonl > $OUT/bench_bj_$TAG.log 2>&1
timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline \
    --parity none --out $OUT/bench_n4032_$TAG.jsonl > $OUT/bench_n4032_$TAG.log 2>&1
timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline \
    --parity none --precond block_jacobi --out $OUT/bench_n4032_bj_$TAG.jsonl > $OUT/bench_n4032_bj_$TAG.log 2>&1
timeout 900 python bench.py --solver banded --steps 5 --warmup 2 --cpu-seconds 3 \
    --out $OUT/bench_banded_$TAG.jsonl > $OUT/bench_banded_$TAG.log 2>&1
bash tools/r2_table2.sh $TAG
timeout 600 python tools/iter_sensitivity.py --gpu --n 1000 --out $OUT/iter_sensitivity_$TAG.json \
    > $OUT/iter_sensitivity_$TAG.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $tool python tools/sanitize_cases.py (SAN_BATCH=3)" >> $OUT/sanitizer_$TAG.txt
  SAN_BATCH=3 timeout 1200 compute-sanitizer --tool $tool python tools/sanitize_cases.py \
      >> $OUT/sanitizer_$TAG.txt 2>&1
  echo "rc=$?" >> $OUT/sanitizer_$TAG.txt
done
for mode in 0 1 2 3; do
  timeout 300 compute-sanitizer --tool racecheck tools/cluster_race_probe $mode > $OUT/race_probe_${TAG}_$mode.txt 2>&1
done
echo done
