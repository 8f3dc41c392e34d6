#!/bin/bash
# Table II analogue: warp efficiency, L1/L2 hit rates, HBM
# throughput of the solve kernel per format x placement, + bench lines.
set -u
TAG=${1:-t2}
OUT=gpurun_out; mkdir -p $OUT
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__thread_inst_executed_per_inst_executed.ratio,l1tex__t_sector_hit_rate.pct,lts__t_sector_hit_rate.pct,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread
: > $OUT/table2_$TAG.txt
for cfg in "ell auto" "csr auto" "ell stream" "csr stream" "ell smem" "csr smem"; do
  set -- $cfg
  timeout 600 python bench.py --format $1 --placement $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
      --parity none --out $OUT/bench_${TAG}_$1_$2.jsonl > /dev/null 2>&1
  timeout 600 ncu --metrics $M --clock-control none --csv -k regex:bicgstab -s 3 -c 1 \
      python bench.py --format $1 --placement $2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
      --parity none > $OUT/ncu_${TAG}_$1_$2.csv 2>&1
  echo "== $1 $2" >> $OUT/table2_$TAG.txt
done
echo done
