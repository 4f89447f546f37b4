"""Aggregate an ncu --csv capture with dram__bytes_{read,write}.sum and
gpu__time_duration.sum per launch into profiles/ncu_summary.json (per-kernel mean DRAM
bytes and time per launch, and each kernel's share of the step)."""
import csv, sys, json, collections, os
path, out = sys.argv[1], sys.argv[2]
with open(path) as f:
    lines = [l for l in f if l.startswith('"')]
per = collections.defaultdict(lambda: collections.defaultdict(float))
for r in csv.DictReader(lines):
    name = r["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("eclscc::", "")
    key = (name, r["ID"])
    v = float(r["Metric Value"].replace(",", "") or 0)
    u = r.get("Metric Unit", "")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3, "us": 1,
             "usecond": 1, "ms": 1e3, "msecond": 1e3}.get(u, 1)
    per[key][r["Metric Name"]] += v * scale
agg = collections.defaultdict(lambda: {"launches": 0, "dram_bytes": 0.0, "time_us": 0.0})
for (name, _), m in per.items():
    a = agg[name]
    a["launches"] += 1
    a["dram_bytes"] += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
    a["time_us"] += m.get("gpu__time_duration.sum", 0)
tot = sum(a["time_us"] for a in agg.values()) or 1
res = {"source": os.path.basename(path), "note": "ncu, cold-cache serialised launches of one ecl_scc run; compare shares, not absolutes",
       "kernels": {}}
for name, a in sorted(agg.items(), key=lambda kv: -kv[1]["time_us"]):
    res["kernels"][name] = {"launches": a["launches"], "dram_bytes_per_launch": round(a["dram_bytes"] / a["launches"]),
                            "time_us_per_launch": round(a["time_us"] / a["launches"], 2),
                            "share_of_step": round(a["time_us"] / tot, 4),
                            "dram_gbs": round(a["dram_bytes"] / (a["time_us"] * 1e-6) / 1e9, 1) if a["time_us"] else None}
json.dump(res, open(out, "w"), indent=1)
for k, v in res["kernels"].items():
    print(f"{k:24s} {v}")
