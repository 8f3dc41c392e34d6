"""Summarise an ncu --set full report of the solve kernel (key metrics)."""
import csv, subprocess, sys
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
h, units, vals = rows[0], rows[1], rows[2]
d = dict(zip(h, vals))
keys = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "memory_l1_wavefronts_shared", "memory_l1_wavefronts_shared_ideal",
        "smsp__sass_inst_executed_op_shared_ld.sum", "smsp__sass_inst_executed_op_shared_st.sum",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__thread_inst_executed_per_inst_executed.ratio",
        "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum"]
for k in keys:
    if k in d:
        print(f"{k:80s} {units[h.index(k)]:>10s} {d[k]}")
stalls = [k for k in h if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio")]
tot = sum(float(d[k] or 0) for k in stalls)
print("stall breakdown (warp-cycles per issued instruction):")
for k in sorted(stalls, key=lambda k: -float(d[k] or 0))[:8]:
    print(f"   {k.replace('smsp__average_warps_issue_stalled_','').replace('_per_issue_active.ratio',''):28s} {float(d[k]):.3f}")
