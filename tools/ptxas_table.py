import re, sys
lines = open(sys.argv[1]).read().split('\n')
cur=None
for l in lines:
    m = re.search(r"Compiling entry function '(\S+)'", l)
    if m: cur = m.group(1); spill=''; continue
    m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", l)
    if m and cur: spill = f"spill {m.group(1)}/{m.group(2)}"
    m = re.search(r"Used (\d+) registers", l)
    if m and cur:
        k = re.search(r"bicgstab_kernelILi(\d)ELi(\d)ELi(\d+)ELb[01]ELi(\d)ELi(\d+)", cur)
        if k: print(f"fmt={k.group(1)} place={k.group(2)} WB={k.group(3)} R={k.group(4)} NT={k.group(5)}: regs {m.group(1)} {spill}")
        cur=None
