"""Asynchronous Phase-2 policies on the CPU model (tools/sim/asyncsim.cpp)."""
import ctypes, os, sys, time
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from simlib import gen, prio
L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libasyncsim.so"))
L.asyncsim.restype = ctypes.c_int64
P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 70
g = gen.mesh(N, gen.ordinate(0), seed=4, order="blocked8", **gen.C4_MESH)
pr = prio(g.n).astype(np.int32)
tiles = (np.arange(g.n) // 2048).astype(np.int32)
nt = int(tiles.max()) + 1
for W in (max(1, nt // 18),):
    for pol in (0, 1, 2, 3, 4, 6, 8):
        out = np.zeros(3, dtype=np.int64); t = time.time()
        L.asyncsim(ctypes.c_int32(g.n), P(g.row_ptr), P(g.col_idx), P(tiles), ctypes.c_int32(nt), P(pr), ctypes.c_int32(W), ctypes.c_int32(pol), P(out))
        print(f"N={N} tiles={nt} W={W:4d} policy={pol} rounds={out[0]:6d} visits/tile={out[1]/nt:6.1f} raises/n={out[2]/g.n:5.1f} ({time.time()-t:.1f}s)", flush=True)
