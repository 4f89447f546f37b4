"""One ecl_scc run between cudaProfilerStart/Stop (for ncu --profile-from-start off)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_sc_alabandisbb23_b200 as E

cfg = sys.argv[1] if len(sys.argv) > 1 else "c4"
order = sys.argv[2] if len(sys.argv) > 2 else "blocked8"
g = gen.config(cfg, order=order) if cfg in ("c2", "c4") else gen.config(cfg)
rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
lab = torch.empty(g.n, dtype=torch.int32, device="cuda")
plan = E.Plan(g.n, g.nnz, E.NO_VALIDATE)
_, st = E.ecl_scc(rp, ci, lab, plan=plan, stats=True)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
_, st = E.ecl_scc(rp, ci, lab, plan=plan, stats=True)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print({k: v for k, v in st.items() if k not in ("edges_kept",)})
c = plan.counters()
print('counters [visits, block_rounds, warp_drains, vertex_pushes]:', c[:4])
if c[0]: print('cycles per visit: step1 %.0f step2 %.0f step3 %.0f; raised vertex-dirs per visit %.0f' % (c[4]/c[0], c[5]/c[0], c[6]/c[0], c[7]/c[0]))
if os.environ.get("PROF_PROTO") and c[0]: print('protocol cycles per visit: claim %.0f visit %.0f fences+marks+finish %.0f' % (c[4]/c[0], c[5]/c[0], c[6]/c[0]))
