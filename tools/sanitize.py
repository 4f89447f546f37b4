"""Workload for compute-sanitizer (memcheck / racecheck / synccheck): every entry point of the
C ABI on small inputs (C1 G(n,m), the worked example, a small curved mesh, a small R-MAT),
labels checked against the oracle.  Usage (GPU box):
    compute-sanitizer --tool memcheck python tools/sanitize.py [small]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import gen
import oracle
import paper_conf_sc_alabandisbb23_b200 as E

small = len(sys.argv) > 1 and sys.argv[1] == "small"
graphs = [gen.appendix_a(), gen.config("c1"), gen.mesh(8 if small else 16, gen.ordinate(3), seed=4, **gen.C4_MESH)]
if not small:
    graphs.append(gen.rmat(12, 16, seed=3))
for g in graphs:
    rp, ci = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda()
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    for fl in (0, E.NO_ASYNC, E.IDENTITY_IDS | E.TRIM2, E.FOUR_SIG):
        lab = E.ecl_scc(rp, ci, plan=E.Plan(g.n, g.nnz, fl))
        torch.cuda.synchronize()
        assert np.array_equal(lab.cpu().numpy(), truth), (g.name, fl)
    lv, d = E.ecl_scc_levels(rp, ci, lab)
    lab2 = E.ecl_scc_partitioned_emulated(2, rp, ci)
    torch.cuda.synchronize()
    assert np.array_equal(lab2.cpu().numpy(), truth), g.name
    print("ok", g.name, "depth", d, flush=True)
labs = E.ecl_scc_batched([(torch.from_numpy(h.row_ptr).cuda(), torch.from_numpy(h.col_idx).cuda()) for h in graphs])
torch.cuda.synchronize()
for h, l in zip(graphs, labs):
    assert np.array_equal(l.cpu().numpy(), oracle.tarjan_labels(h.row_ptr, h.col_idx))
hl = E.ecl_scc_batched_host([(torch.from_numpy(h.row_ptr).pin_memory(), torch.from_numpy(h.col_idx).pin_memory())
                             for h in graphs])
for h, l in zip(graphs, hl):
    assert np.array_equal(l.numpy(), oracle.tarjan_labels(h.row_ptr, h.col_idx))
print("sanitize workload ok", flush=True)
