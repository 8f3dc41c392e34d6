"""Per-source-line warp-stall samples of one kernel in an ncu --set full report
(--import-source on, -lineinfo build):  python tools/ncu_lines.py rep.ncu-rep [top]
Prints the lines with the most stall samples and their dominant stall reasons."""
import csv
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
fname, hdr, agg = None, None, []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r[0]:
        continue  # SASS rows (empty line number)
    d = dict(zip(hdr[2:], r[2:]))
    try:
        samples = int(d.get("Warp Stall Sampling (All Samples)", "0") or 0)
    except ValueError:
        continue
    stalls = {k: int(v) for k, v in d.items() if k.startswith("stall_") and "Not Issued" not in k
              and v not in ("", "-") and v.isdigit()}
    agg.append((samples, fname, r[0], r[1][:70], stalls))
tot = sum(a[0] for a in agg) or 1
agg.sort(key=lambda a: -a[0])
print(f"total samples {tot}")
for s, f, ln, src, st in agg[:top]:
    best = sorted(st.items(), key=lambda kv: -kv[1])[:3]
    print(f"{100 * s / tot:5.1f}% {f}:{ln:<5s} {src:70s} " +
          " ".join(f"{k[6:]}={100 * v / max(s, 1):.0f}%" for k, v in best))
