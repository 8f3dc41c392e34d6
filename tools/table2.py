"""Table II analogue from tools/r2_table2.sh outputs:
per format x placement: throughput, warp efficiency, L1/L2 hit rates, HBM."""
import csv
import glob
import json
import os
import sys

tag = sys.argv[1]
g = "gpurun_out"
print(f"{'format':6s} {'placement':9s} {'M sys/s':>8s} {'kernel ms':>9s} {'warp eff %':>10s} "
      f"{'L1 hit %':>8s} {'L2 hit %':>8s} {'HBM GB/s':>9s} {'SMEM pipe %':>11s} {'FP64 %':>7s} "
      f"{'warps act %':>11s} {'regs':>4s}  kernel")
for fmt, pl in (("ell", "auto"), ("csr", "auto"), ("ell", "stream"), ("csr", "stream"),
                ("ell", "smem"), ("csr", "smem")):
    try:
        b = json.loads(open(f"{g}/bench_{tag}_{fmt}_{pl}.jsonl").read().strip().splitlines()[-1])
        allr = list(csv.reader(open(f"{g}/ncu_{tag}_{fmt}_{pl}.csv")))
        i0 = next(i for i, r in enumerate(allr) if r and r[0] == "ID")
        rows = [allr[i0]] + [r for r in allr[i0 + 1:] if len(r) == len(allr[i0])]
        h = rows[0]
        m = {r[h.index("Metric Name")]: (r[h.index("Metric Value")], r[h.index("Metric Unit")])
             for r in rows[1:]}
        kern = rows[1][h.index("Kernel Name")]
    except Exception as e:  # noqa: BLE001
        print(fmt, pl, "missing", e)
        continue
    def f(k):
        v, u = m[k]
        return float(v.replace(",", "")) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1,
                                             "ms": 1e-3, "us": 1e-6, "ns": 1e-9}.get(u, 1)
    t = f("gpu__time_duration.sum")
    hbm = (f("dram__bytes_read.sum") + f("dram__bytes_write.sum")) / t / 1e9
    print(f"{fmt:6s} {pl:9s} {b['value'] / 1e6:8.3f} {t * 1e3:9.3f} "
          f"{100 * f('smsp__thread_inst_executed_per_inst_executed.ratio') / 32:10.1f} "
          f"{f('l1tex__t_sector_hit_rate.pct'):8.1f} {f('lts__t_sector_hit_rate.pct'):8.1f} "
          f"{hbm:9.0f} {f('l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed'):11.1f} "
          f"{f('sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active'):7.1f} "
          f"{f('sm__warps_active.avg.pct_of_peak_sustained_active'):11.1f} "
          f"{int(f('launch__registers_per_thread')):4d}  {kern[:60]}")
