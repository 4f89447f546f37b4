"""One batched ecl_scc run over the 64-graph C5 workload between cudaProfilerStart/Stop (for
ncu --profile-from-start off)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_sc_alabandisbb23_b200 as E

graphs = [gen.config("c5one", order="blocked8", d=d) for d in range(64)]
dg = [(torch.from_numpy(h.row_ptr).cuda(), torch.from_numpy(h.col_idx).cuda()) for h in graphs]
labs = [torch.empty(h.n, dtype=torch.int32, device="cuda") for h in graphs]
plan = E.Plan(sum(h.n for h in graphs), sum(h.nnz for h in graphs), E.NO_VALIDATE)
E.ecl_scc_batched(dg, labs, plan=plan)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
_, st = E.ecl_scc_batched(dg, labs, plan=plan, stats=True)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print({k: v for k, v in st.items() if k in ("iterations", "passes", "kernel_launches")})
