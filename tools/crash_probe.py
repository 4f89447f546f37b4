"""Run ecl_scc on a few configs, report status (for compute-sanitizer runs)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, gen, oracle, numpy as np
import paper_conf_sc_alabandisbb23_b200 as E
for name in sys.argv[1:]:
    if name.startswith("mesh"):
        N, order = int(name.split(":")[1]), name.split(":")[2]
        g = gen.mesh(N, gen.ordinate(0), seed=4, order=order, **gen.C4_MESH)
    else:
        g = gen.config(name, order="lex")
    rp = torch.from_numpy(g.row_ptr).cuda(); ci = torch.from_numpy(g.col_idx).cuda()
    try:
        lab = E.ecl_scc(rp, ci); torch.cuda.synchronize()
        ok = np.array_equal(lab.cpu().numpy(), oracle.tarjan_labels(g.row_ptr, g.col_idx))
        print(name, "ok" if ok else "WRONG", flush=True)
    except Exception as e:
        print(name, "ERROR", e, flush=True); break
