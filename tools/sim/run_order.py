"""Tile dispatch order x concurrency window (CPU model)."""
import os, sys, time
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from simlib import run, gen, prio, mesh_coords, blocked_tiles
N = int(sys.argv[1]) if len(sys.argv) > 1 else 70
g = gen.mesh(N, gen.ordinate(0), seed=4, order="lex", **gen.C4_MESH)
n = g.n
v, x, y, z = mesh_coords(N, n)
tile_of = blocked_tiles(N, g)
nt = int(tile_of.max()) + 1
om = np.array(gen.ordinate(0))
cnt = np.bincount(tile_of, None, nt)
proj = (om[0] * np.bincount(tile_of, x, nt) + om[1] * np.bincount(tile_of, y, nt) + om[2] * np.bincount(tile_of, z, nt)) / cnt
orders = {"index": None, "omega-projection": np.argsort(proj).astype(np.int32)}
rand = prio(n).astype(np.int32)
for oname, od in orders.items():
    for W in [int(w) for w in os.environ.get("WINDOWS", "1,64,444,100000").split(",")]:
        t0 = time.time()
        out = run(g, tile_of, rand, gs=1, order=od, window=W)
        print(f"order={oname:17s} window={W:6d} passes={out[0]:3d} visited/n={out[2]/n:5.1f} raises/n={out[3]/n:5.2f} ({time.time()-t0:.1f}s)", flush=True)
