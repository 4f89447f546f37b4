"""Device time of the edge-partitioned mode with P emulated ranks on one GPU (development
helper): the same per-rank kernels and exchange protocol as the NCCL mode, the all-reduce
replaced by an element-wise reduction over the P replicas."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import gen
import paper_conf_sc_alabandisbb23_b200 as E

for c in sys.argv[1:] or ["c2", "c4"]:
    g = gen.config(c, order="blocked8")
    rp, ci = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda()
    for P in (1, 2, 4, 8):
        E.ecl_scc_partitioned_emulated(P, rp, ci)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        _, st = E.ecl_scc_partitioned_emulated(P, rp, ci, stats=True)
        b.record()
        torch.cuda.synchronize()
        t = a.elapsed_time(b)
        print(f"{c} P={P}: {t:.1f} ms ({g.nnz / t / 1e3:.0f} Medges/s), iterations={st['iterations']} "
              f"local passes={st['passes']}", flush=True)
