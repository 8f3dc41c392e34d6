"""SASS opcode histogram of one kernel of an object file (cuobjdump):
  python tools/sass_hist.py paper_conf_ipps_kashinksla22_b200/build_obj/k_line.o bicgstab_line3_kernelILi32ELi2E"""
import collections
import re
import subprocess
import sys

obj, pat = sys.argv[1], sys.argv[2]
out = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s+Function : ", out)
for f in funcs[1:]:
    name = f.split("\n", 1)[0].strip()
    if pat not in name:
        continue
    ops = collections.Counter()
    for line in f.split("\n"):
        m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]+)", line)
        if m:
            ops[m.group(1)] += 1
    tot = sum(ops.values())
    print(f"kernel {name}\ninstructions {tot}")
    for op, c in ops.most_common():
        print(f"{c:6d}  {op}")
    break
