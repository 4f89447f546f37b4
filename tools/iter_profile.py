"""Per-outer-iteration device times (ECL_SCC_TIME_STAGES) on the BASELINE configs (development helper)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import gen
import paper_conf_sc_alabandisbb23_b200 as E


def run(name, g, flags=0, reps=3):
    rp = torch.from_numpy(g.row_ptr).cuda()
    ci = torch.from_numpy(g.col_idx).cuda()
    plan = E.Plan(g.n, g.nnz, flags | E.NO_VALIDATE | E.TIME_STAGES)
    lab = torch.empty(g.n, dtype=torch.int32, device="cuda")
    E.ecl_scc(rp, ci, lab, plan=plan)
    best = None
    for _ in range(reps):
        _, st = E.ecl_scc(rp, ci, lab, plan=plan, stats=True)
        if best is None or st["ms_prop"] + st["ms_compact"] < best["ms_prop"] + best["ms_compact"]:
            best = st
    st = best
    print(f"== {name} n={g.n} m={g.nnz} ingest={st['ms_ingest']:.3f} compact={st['ms_compact']:.3f} "
          f"prop={st['ms_prop']:.3f} iters={st['iterations']} launches={st['kernel_launches']}")
    for k in range(len(st["edges_in"])):
        print(f"  it{k+1:2d} V={st['vertices_in'][k]:9d} E={st['edges_in'][k]:9d} passes={st['passes_iter'][k]:4d} "
              f"compact={st['ms_compact_iter'][k]:7.3f} prop={st['ms_prop_iter'][k]:7.3f}")
    if len(st["ms_compact_iter"]) > len(st["edges_in"]):
        print(f"  final compact={st['ms_compact_iter'][-1]:.3f}")
    sys.stdout.flush()


if __name__ == "__main__":
    which = sys.argv[1:] or ["c4", "c3", "c2"]
    for w in which:
        if w in ("c2", "c4"):
            for order in ("blocked8", "lex"):
                run(f"{w} {order}", gen.config(w, order=order))
        else:
            run(w, gen.config(w))
