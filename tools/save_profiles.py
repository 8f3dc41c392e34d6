"""Copy a gpu_profile.sh run (tag) into profiles/: launch list + summary,
ncu summary of the solve kernel, bench line, ncu traffic for bench.py."""
import csv, json, shutil, subprocess, sys
tag, out = sys.argv[1], sys.argv[2]          # e.g. r1v5 r1
g = "gpurun_out"
shutil.copy(f"{g}/launches_{tag}.csv", f"profiles/{out}_launches.csv")
with open(f"profiles/{out}_launches_summary.txt", "w") as f:
    f.write(subprocess.run([sys.executable, "tools/launch_summary.py", f"{g}/launches_{tag}.csv"],
                           capture_output=True, text=True).stdout)
shutil.copy(f"{g}/bench_{tag}.jsonl", f"profiles/{out}_bench.jsonl")
rep = f"{g}/prof_{tag}.ncu-rep"
with open(f"profiles/{out}_ncu_solve_kernel.txt", "w") as f:
    f.write(f"# ncu --set full --clock-control none, bench.py default workload ({tag})\n")
    f.write(subprocess.run([sys.executable, "tools/ncu_summary.py", rep], capture_output=True,
                           text=True).stdout)
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
d, u = dict(zip(rows[0], rows[2])), dict(zip(rows[0], rows[1]))
def val(k):
    return float(d[k].replace(",", "")) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3}.get(u[k], 1)
name = d.get("Kernel Name", "bicgstab_kernel")
bench = json.loads(open(f"{g}/bench_{tag}.jsonl").read().strip().splitlines()[-1])
t = {"source": f"ncu --set full --clock-control none, one launch of {name} (bench.py default "
               f"workload: 1e5 systems, 992 rows, x0 = 0), capture {tag}",
     "kernel": name, "systems_per_launch": bench["config"]["batch_per_gpu"],
     "dram_bytes_read": val("dram__bytes_read.sum"), "dram_bytes_write": val("dram__bytes_write.sum"),
     "smem_data_pipe_wavefronts": val("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
     "duration_ms": val("gpu__time_duration.sum")}
for key, metric in (("smem_pipe_busy", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed"),
                    ("fp64_pipe_busy", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
                    ("lsu_pipe_busy", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"),
                    ("warps_active", "sm__warps_active.avg.pct_of_peak_sustained_active")):
    if metric in d:
        t[key] = float(d[metric].replace(",", "")) / 100.0
if "launch__registers_per_thread" in d:
    t["registers_per_thread"] = int(float(d["launch__registers_per_thread"]))
t["dram_bytes_per_launch"] = t["dram_bytes_read"] + t["dram_bytes_write"]
t["smem_data_pipe_bytes_per_launch"] = t["smem_data_pipe_wavefronts"] * 128
json.dump(t, open("profiles/ncu_traffic.json", "w"), indent=1)
print(json.dumps(t, indent=1))
