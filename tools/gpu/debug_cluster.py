import os, sys, random
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import gen, oracle
import paper_conf_sc_alabandisbb23_b200 as E
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
from prio_ref import prio

def relabel(g, pi):
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    return gen.from_edges(g.n, np.stack([pi[src], pi[g.col_idx]], 1))

rng = random.Random(7)
for n in (3000, 5000, 9000):
    k = 3 * n
    src = np.array([rng.randrange(n) for _ in range(k)], dtype=np.int64)
    dst = np.clip(src + np.array([rng.randrange(-3000, 3000) for _ in range(k)]), 0, n - 1)
    g = gen.from_edges(n, np.stack([src, dst], 1))
    rp, ci = torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda()
    for fl in (E.IDENTITY_IDS, E.IDENTITY_IDS | E.CLUSTER, E.IDENTITY_IDS | E.NO_TRIM | E.CLUSTER):
        trim = not (fl & E.NO_TRIM)
        s = oracle.ecl_scc(g.row_ptr, g.col_idx, trim=trim, snap_iter=1)
        gi, go, st = E.ecl_scc_debug_run(rp, ci, 1, flags=fl)
        gi, go = gi.cpu().numpy(), go.cpu().numpy()
        di = np.nonzero(gi != s.snap_in)[0]; do = np.nonzero(go != s.snap_out)[0]
        print(f"n={n} flags={hex(fl)} in-diff={len(di)} out-diff={len(do)}", flush=True)
        for v in di[:5]:
            print(f"   in  v={v} half={(v // 2048) % 2} pair={v // 4096} gpu={gi[v]} oracle={s.snap_in[v]}")
        for v in do[:5]:
            print(f"   out v={v} half={(v // 2048) % 2} pair={v // 4096} gpu={go[v]} oracle={s.snap_out[v]}")
