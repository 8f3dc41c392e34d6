set -u
OUT=gpurun_out; mkdir -p $OUT; TAG=gmg
timeout 1200 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_gpu_$TAG.log
: > $OUT/summary_$TAG.txt
for g in "32 31" "40 25"; do
  set -- $g
  for gk in 0 1; do
  BSOLVE_LINE_GENERIC=$gk timeout 600 python bench.py --nx $1 --ny $2 --solver gmres --steps 5 --warmup 2 --no-e2e --no-cpu-baseline \
     --parity none > $OUT/bench_${TAG}_$1x$2_$gk.log 2>&1
  tail -1 $OUT/bench_${TAG}_$1x$2_$gk.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('gmres $1x$2 generic=$gk', round(d['value']/1e6,3), d['plan'].get('line_generic'), d['plan'].get('kernel_mode'))" >> $OUT/summary_$TAG.txt 2>&1
  done
done
cat $OUT/summary_$TAG.txt; tail -3 $OUT/pytest_gpu_$TAG.log
