"""Aggregate an ncu --csv launch capture of one ecl_scc run (gpu__time_duration.sum,
dram__bytes_{read,write}.sum, the L2 atomic / reduction request counters, hit rates, warps
active) per kernel into profiles/ncu_summary.json under configs[<key>] (per-launch means,
each kernel's share of the step).  bench.py reads roofline.traffic from there, for the
config it measures.

    python tools/ncu_traffic.py gpurun_out/ncu_c4.csv c4/blocked8 profiles/ncu_summary.json"""
import collections
import csv
import json
import os
import sys

path, key, out = sys.argv[1], sys.argv[2], sys.argv[3]
with open(path) as f:
    lines = [l for l in f if l.startswith('"')]
per = collections.defaultdict(lambda: collections.defaultdict(float))
for r in csv.DictReader(lines):
    name = r["Kernel Name"].split("(")[0].split("<")[0].replace("void ", "").replace("eclscc::", "")
    v = float(r["Metric Value"].replace(",", "") or 0)
    u = r.get("Metric Unit", "")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3, "us": 1,
             "usecond": 1, "ms": 1e3, "msecond": 1e3}.get(u, 1)
    per[(name, r["ID"])][r["Metric Name"]] += v * scale
SUMS = {"lts__t_requests_srcunit_tex_op_atom.sum": "l2_atom_requests",
        "lts__t_requests_srcunit_tex_op_red.sum": "l2_red_requests"}
MEANS = {"lts__t_sector_hit_rate.pct": "l2_hit_pct", "l1tex__t_sector_hit_rate.pct": "l1_hit_pct",
         "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
         "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct"}
agg = collections.defaultdict(lambda: collections.defaultdict(float))
for (name, _), m in per.items():
    a = agg[name]
    a["launches"] += 1
    a["dram_bytes"] += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
    a["time_us"] += m.get("gpu__time_duration.sum", 0)
    for k, nm in SUMS.items():
        a[nm] += m.get(k, 0)
    for k, nm in MEANS.items():   # time-weighted
        a[nm] += m.get(k, 0) * m.get("gpu__time_duration.sum", 0)
tot = sum(a["time_us"] for a in agg.values()) or 1
res = {"source": os.path.basename(path),
       "note": "ncu, one ecl_scc run, cold-cache serialised launches: compare shares, not absolutes",
       "kernels": {}}
for name, a in sorted(agg.items(), key=lambda kv: -kv[1]["time_us"]):
    L, T = a["launches"], a["time_us"] or 1e-9
    res["kernels"][name] = {
        "launches": int(L), "dram_bytes_per_launch": round(a["dram_bytes"] / L),
        "time_us_per_launch": round(a["time_us"] / L, 2), "share_of_step": round(a["time_us"] / tot, 4),
        "dram_gbs": round(a["dram_bytes"] / (T * 1e-6) / 1e9, 1),
        **{nm: round(a[nm] / L) for nm in SUMS.values()},
        **{nm: round(a[nm] / T, 1) for nm in MEANS.values()}}
try:
    allres = json.load(open(out))
    if "configs" not in allres:
        allres = {"configs": {}}
except Exception:
    allres = {"configs": {}}
allres["configs"][key] = res
json.dump(allres, open(out, "w"), indent=1)
for k, v in list(res["kernels"].items())[:12]:
    print(f"{k:24s} {v}")
