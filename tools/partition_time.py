"""Device time of the edge-partitioned (halo) mode with P emulated ranks on one GPU
(development helper).  The P ranks run one after another on one device with the same kernels
and exchange protocol as the NCCL mode (the all-reduces are reductions over the P buffers,
the fused pushes target the P halo buffers), with workspaces allocated beforehand, so the
time is ~ the sum of the ranks' work plus the exchanges -- not a multi-GPU time."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import gen
import paper_conf_sc_alabandisbb23_b200 as E

for c in sys.argv[1:] or ["c2", "c4"]:
    g = gen.config(c, order="blocked8")
    rp, ci = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda()
    lab = torch.empty(g.n, dtype=torch.int32, device="cuda")
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    plan = E.Plan(g.n, g.nnz, E.NO_VALIDATE)
    E.ecl_scc(rp, ci, lab, plan=plan)
    a.record()
    E.ecl_scc(rp, ci, lab, plan=plan)
    b.record()
    torch.cuda.synchronize()
    print(f"{c} single GPU: {a.elapsed_time(b):.2f} ms", flush=True)
    for P in (1, 2, 4, 8):
        for fl, nm in ((0, "fused pushes"), (E.HALO_ALLREDUCE, "all-reduce exchange")):
            ep = E.EmulatedPlan(P, rp, g.nnz, fl)
            E.ecl_scc_partitioned_emulated(P, rp, ci, flags=fl, plan=ep)
            a.record()
            _, st = E.ecl_scc_partitioned_emulated(P, rp, ci, stats=True, flags=fl, plan=ep)
            b.record()
            torch.cuda.synchronize()
            t = a.elapsed_time(b)
            print(f"{c} P={P} {nm:20s}: {t:7.1f} ms  iterations={st['iterations']} exchange rounds={st['passes']} "
                  f"collectives={st['exchanges']} comm bytes={st['comm_bytes']} ms_comm={st['ms_comm']:.2f}",
                  flush=True)
