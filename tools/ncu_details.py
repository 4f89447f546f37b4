"""Flatten `ncu -i X --page details --csv` into one line per metric (development helper)."""
import csv, sys
title = sys.argv[1] if len(sys.argv) > 1 else ""
if title:
    print(title)
for r in csv.DictReader(sys.stdin):
    if not r.get("Metric Name"):
        continue
    k = r["Kernel Name"].split("(")[0]
    print(f'{r["ID"]:>3} {k[:14]:14s} {r["Section Name"][:26]:26s} {r["Metric Name"][:44]:44s} '
          f'{r["Metric Unit"][:14]:14s} {r["Metric Value"]}')
