#!/bin/bash
set -u
TAG=${1:-bj}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_blockjacobi.py tests/test_gpu_parity.py -x -q > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --parity sample --cpu-seconds 3 --out $OUT/bench_${TAG}_jacobi.jsonl > $OUT/bench_${TAG}_jacobi.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --parity sample --cpu-seconds 3 --precond block_jacobi --out $OUT/bench_${TAG}_bj.jsonl > $OUT/bench_${TAG}_bj.log 2>&1
echo done
