"""Device time of ecl_scc_levels (sweep levels of the condensation) after ecl_scc on the
BASELINE configs (development helper)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import gen
import paper_conf_sc_alabandisbb23_b200 as E

for c in sys.argv[1:] or ["c2", "c3", "c4"]:
    if c.startswith("mesh"):                 # meshN: a C4-like mesh of N^3 cubes, blocked8
        g = gen.mesh(int(c[4:]), gen.ordinate(0), seed=4, order="blocked8", **gen.C4_MESH)
    else:
        g = gen.config(c, order="blocked8") if c in ("c2", "c4", "c5one") else gen.config(c)
    rp, ci = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda()
    plan = E.Plan(g.n, g.nnz, E.NO_VALIDATE)
    lab = E.ecl_scc(rp, ci, plan=plan)
    lv = torch.empty_like(lab)
    for name, p in (("default", plan), ("kahn", E.Plan(g.n, g.nnz, E.NO_VALIDATE | E.NO_ASYNC))):
        E.ecl_scc_levels(rp, ci, lab, lv, plan=p)
        ts = []
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            _, depth = E.ecl_scc_levels(rp, ci, lab, lv, plan=p)
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        t = float(np.median(ts))
        print(f"{c} {name}: n={g.n} nnz={g.nnz} depth={depth} levels {t:.3f} ms ({g.nnz / t / 1e3:.0f} Medges/s, "
              f"{t / max(depth, 1) * 1e3:.2f} us per level)", flush=True)
