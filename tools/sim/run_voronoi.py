"""BFS-Voronoi storage clustering vs ID-range tiles (CPU model)."""
import os, sys, time
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from simlib import run, gen, prio, blocked_tiles
import scipy.sparse as sp

def voronoi_order(g, K_every=2048, seed=1):
    n = g.n
    src = np.repeat(np.arange(n), np.diff(g.row_ptr)); dst = g.col_idx
    A = sp.csr_matrix((np.ones(len(src), np.int8), (src, dst)), shape=(n, n))
    A = (A + A.T).tocsr()
    rng = np.random.default_rng(seed)
    seeds = np.sort(rng.choice(n, n // K_every, replace=False))
    lab = np.full(n, -1, np.int64); lab[seeds] = np.arange(len(seeds))
    rounds = 0
    while (lab < 0).any():
        rounds += 1
        # each unlabeled vertex takes the min label among labeled neighbours
        m = np.where(lab >= 0, lab, np.iinfo(np.int64).max)
        nbmin = np.full(n, np.iinfo(np.int64).max)
        rows = np.repeat(np.arange(n), np.diff(A.indptr))
        np.minimum.at(nbmin, rows, m[A.indices])
        upd = (lab < 0) & (nbmin < np.iinfo(np.int64).max)
        if not upd.any(): lab[lab < 0] = len(seeds); break
        lab[upd] = nbmin[upd]
    order = np.lexsort((np.arange(n), lab))      # by cluster, then id
    pos = np.empty(n, np.int64); pos[order] = np.arange(n)
    return pos, rounds, np.bincount(lab)

N = int(sys.argv[1]) if len(sys.argv) > 1 else 70
pr = None
for order in ("lex", "blocked8"):
    g = gen.mesh(N, gen.ordinate(0), seed=4, order=order, **gen.C4_MESH)
    pr = prio(g.n).astype(np.int32)
    t0 = time.time(); pos, rounds, sizes = voronoi_order(g)
    tv = (pos // 2048).astype(np.int32)
    o1 = run(g, (np.arange(g.n) // 2048).astype(np.int32), pr)
    o2 = run(g, tv, pr)
    print(f"{order:9s} id-ranges: passes={o1[0]} visited/n={o1[2]/g.n:.1f} | voronoi(rounds={rounds}, size mean {sizes.mean():.0f} sd {sizes.std():.0f}): passes={o2[0]} visited/n={o2[2]/g.n:.1f}  ({time.time()-t0:.1f}s)", flush=True)
