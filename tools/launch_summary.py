"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV):
per-kernel launch count, total and mean time, share of GPU time."""
import csv, sys, collections
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, vi, mi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name")
agg = collections.OrderedDict()
for r in rows[1:]:
    if r[mi] != "gpu__time_duration.sum":
        continue
    name = r[ki]
    t = float(r[vi].replace(",", ""))
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += t
tot = sum(v[1] for v in agg.values())
print(f"{'kernel':70s} {'launches':>8s} {'total ms':>10s} {'mean us':>10s} {'share':>7s}")
for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k[:70]:70s} {c:8d} {t/1e6:10.3f} {t/c/1e3:10.1f} {100*t/tot:6.1f}%")
print(f"{'TOTAL':70s} {sum(v[0] for v in agg.values()):8d} {tot/1e6:10.3f}")
