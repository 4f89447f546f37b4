"""Summarise the quick.sh bench lines and the test tail."""
import glob, json, os
for f in sorted(glob.glob("gpurun_out/q_*.log")):
    for l in open(f):
        if l.startswith("{"):
            d = json.loads(l)
            st = d.get("stages", {})
            print(f"{os.path.basename(f):14s} {d['ms_per_step']:8.2f} ms {d['value']:9.1f} {d['unit']}  frac {d.get('roofline', {}).get('frac')}")
t = open("gpurun_out/pytest_quick.log").read().strip().splitlines()
print(t[-1] if t else "no test log")
