"""Print the per-launch duration sequence of selected kernels from an ncu --csv launch list."""
import csv, sys
path = sys.argv[1]; pat = sys.argv[2] if len(sys.argv) > 2 else "k_prop"
with open(path) as f:
    lines = [l for l in f if l.startswith('"')]
seq = []
for r in csv.DictReader(lines):
    if r.get("Metric Name") != "gpu__time_duration.sum": continue
    name = r["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("eclscc::", "")
    v = float(r["Metric Value"].replace(",", "")); u = r.get("Metric Unit", "ns")
    v = v * (1e3 if u == "usecond" else 1e6 if u == "msecond" else 1)
    seq.append((name, v / 1e3))
line = []
for name, us in seq:
    if name.startswith("k_compact_map"): line.append("|")
    if pat in name: line.append(f"{us:.0f}")
print(" ".join(line))
