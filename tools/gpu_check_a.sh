set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke_a.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke_a.log
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_a.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_a.log
timeout 900 python bench.py --steps 10 --warmup 3 --out $OUT/bench_a.jsonl > $OUT/bench_a.log 2>&1
timeout 600 python bench.py --nx 64 --ny 63 --batch 16384 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --parity none --out $OUT/bench_n4032_a.jsonl > $OUT/bench_n4032_a.log 2>&1
timeout 900 python bench.py --solver banded --steps 5 --warmup 2 --cpu-seconds 3 --out $OUT/bench_banded_a.jsonl > $OUT/bench_banded_a.log 2>&1
echo done
