set -u
OUT=gpurun_out; mkdir -p $OUT; TAG=bjc
timeout 1200 python -m pytest tests/test_gpu_blockjacobi.py tests/test_gpu_parity.py -x -q -k "blockjacobi or cluster" > $OUT/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_$TAG.log
: > $OUT/summary_$TAG.txt
for pc in jacobi block_jacobi; do
  timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 --precond $pc \
     --no-e2e --no-cpu-baseline --parity none > $OUT/bench_${TAG}_$pc.log 2>&1
  tail -1 $OUT/bench_${TAG}_$pc.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['plan']; s=d['solve_stats']; print('$pc', round(d['value']/1e6,3), 'Msys/s', round(d['ms_per_step'],3), 'ms', 'C', p['cluster'], 'it', round(s['iters_mean_ion'],2), round(s['iters_mean_electron'],2), s['all_converged'])" >> $OUT/summary_$TAG.txt 2>&1
done
cat $OUT/summary_$TAG.txt; tail -3 $OUT/pytest_$TAG.log
