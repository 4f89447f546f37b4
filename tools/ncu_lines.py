"""Per-source-line hot spots (stall samples, instructions) from
`ncu -i X --page source --csv --print-source cuda,sass`."""
import csv, sys, io, collections
txt = open(sys.argv[1]).read()
blocks = txt.split('"File Path"')
agg = collections.defaultdict(lambda: [0.0, 0.0, ""])
for b in blocks[1:]:
    lines = b.split("\n")
    path = lines[0].strip(",").strip('"').split("/")[-1]
    body = "\n".join(l for l in lines[1:] if not l.startswith('"Function Name"'))
    rd = csv.reader(io.StringIO(body))
    hdr = next(rd)
    i_line = hdr.index("Line No"); i_samp = hdr.index("Warp Stall Sampling (All Samples)")
    i_inst = hdr.index("Instructions Executed")
    for r in rd:
        if len(r) <= i_inst: continue
        if not r[i_line].strip(): continue     # SASS rows of the cuda,sass listing (already in their line)
        try: samp = float(r[i_samp] or 0); inst = float(r[i_inst] or 0)
        except ValueError: continue
        a = agg[(path, r[i_line])]
        a[0] += samp; a[1] += inst
        if not a[2]: a[2] = r[1].strip()[:90]
tot_s = sum(v[0] for v in agg.values()) or 1; tot_i = sum(v[1] for v in agg.values()) or 1
for (f, ln), (s_, i_, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{100*s_/tot_s:5.1f}% stall  {100*i_/tot_i:5.1f}% inst  {f}:{ln}  {src}")
