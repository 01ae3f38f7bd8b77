"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) by kernel."""
import csv, sys, collections
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
tot = collections.defaultdict(float); cnt = collections.Counter()
for r in rows[1:]:
    if r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
        continue
    name = r[ki].split("(")[0][:60]
    tot[name] += float(r[vi].replace(",", "")); cnt[name] += 1
s = sum(tot.values())
print(f"{'kernel':60s} {'launches':>8s} {'total_us':>10s} {'share':>7s}")
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{k:60s} {cnt[k]:8d} {v/1e3:10.1f} {100*v/s:6.1f}%")
