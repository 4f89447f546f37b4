"""Ablation table in the spirit of the paper's Fig. 14: device time of one ecl_scc
run with each design choice switched off, on C2, C3 and C4 (development helper; the flags are
documented in include/ecl_scc.h and DESIGN.md section 6).

    python tools/ablation.py [c2 c3 c4] > profiles/r01_ablation.txt
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import gen
import paper_conf_sc_alabandisbb23_b200 as E

VARIANTS = [
    ("all optimisations (default)", 0),
    ("no asynchronous Phase 2: one launch per pass (P:192 off)", E.NO_ASYNC),
    ("no tile packs: rows re-walked per visit", E.NO_PACK),
    ("no block-local fixed point: Jacobi passes (P:192 'separate kernels')", E.SYNC_PASSES),
    ("no dirty-tile skipping", E.NO_DIRTY),
    ("raw vertex IDs instead of priorities (the paper's signatures)", E.IDENTITY_IDS),
    ("no Trim-1 (P:83)", E.NO_TRIM),
    ("no storage reordering", E.NO_REORDER),
    ("+ Trim-2 (P:83)", E.TRIM2),
    ("+ 4 signatures (P:194)", E.FOUR_SIG),
    ("+ path compression (P:188)", E.COMPRESS),
    ("+ sound P:190 variant", E.RAISE),
    ("+ cluster pair tiles (DSMEM)", E.CLUSTER),
]


def time_one(g, flags, reps=3, budget_ms=4000.0):
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    plan = E.Plan(g.n, g.nnz, flags | E.NO_VALIDATE)
    lab = torch.empty(g.n, dtype=torch.int32, device="cuda")
    _, st = E.ecl_scc(rp, ci, lab, plan=plan, stats=True)
    ts = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        E.ecl_scc(rp, ci, lab, plan=plan)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
        if ts[-1] > budget_ms:
            break
    return float(np.median(ts)), st


if __name__ == "__main__":
    cfgs = sys.argv[1:] or ["c2", "c3", "c4"]
    for c in cfgs:
        # c2 / c4: lexicographic element IDs; c2b / c4b: 8^3-blocked (the bench default)
        g = gen.config(c[:2], order="blocked8") if c.endswith("b") else gen.config(c)
        base = None
        print(f"== {c}: n={g.n} nnz={g.nnz} ({g.name})", flush=True)
        for name, fl in VARIANTS:
            if c == "c3" and fl in (E.NO_REORDER, E.CLUSTER, E.COMPRESS, E.RAISE):
                continue                      # long rows: pass mode, these do not apply
            t, st = time_one(g, fl)
            base = base or t
            print(f"  {name:70s} {t:9.2f} ms  {g.nnz / t / 1e3:8.1f} Me/s  x{base / t:5.2f}  "
                  f"iters={st['iterations']} passes={st['passes']}", flush=True)
