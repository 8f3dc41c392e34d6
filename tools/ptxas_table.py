"""ptxas register / spill table of every kernel in a verbose build log:
  python -c "from paper_conf_ipps_kashinksla22_b200 import _build; _build.build(force=True, verbose=True)" > build.log
  python tools/ptxas_table.py build.log"""
import re
import subprocess
import sys

rows, cur, spill = [], None, ""
for line in open(sys.argv[1]).read().split("\n"):
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        cur, spill, stack = m.group(1), "", ""
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and cur:
        stack, spill = m.group(1), f"{m.group(2)}/{m.group(3)}"
    m = re.search(r"Used (\d+) registers", line)
    if m and cur:
        rows.append((cur, int(m.group(1)), spill, stack))
        cur = None
names = subprocess.run(["c++filt"], input="\n".join(r[0] for r in rows), capture_output=True,
                       text=True).stdout.split("\n")
seen = set()
print(f"{'regs':>4s} {'spill st/ld B':>13s} {'stack B':>7s}  kernel")
for (mangled, regs, spill, stack), name in sorted(zip(rows, names), key=lambda t: t[1]):
    if name in seen:
        continue
    seen.add(name)
    print(f"{regs:4d} {spill:>13s} {stack:>7s}  {name[:150]}")
