"""Summarise an ncu --csv launch list (gpu__time_duration.sum) by kernel."""
import csv, sys, collections, json
path = sys.argv[1]
rows = []
with open(path) as f:
    lines = [l for l in f if l.startswith('"')]
rd = csv.DictReader(lines)
agg = collections.OrderedDict()
for r in rd:
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    name = r["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("eclscc::", "")
    v = float(r["Metric Value"].replace(",", ""))
    unit = r.get("Metric Unit", "ns")
    if unit == "usecond": v *= 1e3
    elif unit == "msecond": v *= 1e6
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1; a[1] += v
tot = sum(a[1] for a in agg.values())
print(f"{'kernel':28s} {'launches':>8s} {'total_us':>10s} {'share':>7s} {'avg_us':>9s}")
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:28s} {c:8d} {t/1e3:10.1f} {100*t/tot:6.1f}% {t/c/1e3:9.2f}")
print(f"{'TOTAL':28s} {sum(a[0] for a in agg.values()):8d} {tot/1e3:10.1f}")
