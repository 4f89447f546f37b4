"""Evaluate tile shapes / priorities with the CPU model (tools/sim/tilesim.cpp)."""
import ctypes, os, sys, time
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import gen
from prio_ref import prio

L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libtilesim.so"))
L.tilesim.restype = ctypes.c_int64
L.tilesim.argtypes = None
P = lambda a: a.ctypes.data_as(ctypes.c_void_p)

def sim(g, tile_of, pr, heap=0, gs=0):
    tile_of = np.ascontiguousarray(tile_of, dtype=np.int32)
    _, tile_of = np.unique(tile_of, return_inverse=True)
    tile_of = tile_of.astype(np.int32)
    out = np.zeros(4, dtype=np.int64)
    L.tilesim(ctypes.c_int32(g.n), P(g.row_ptr), P(g.col_idx), P(tile_of), ctypes.c_int32(int(tile_of.max()) + 1),
              P(np.ascontiguousarray(pr, dtype=np.int32)), P(out), ctypes.c_int(heap), ctypes.c_int(gs), None, ctypes.c_int32(1))
    return out

if __name__ != '__main__':
    raise SystemExit  # imported for helpers
N = int(sys.argv[1]) if len(sys.argv) > 1 else 70
g = gen.mesh(N, gen.ordinate(0), seed=4, order="lex", **gen.C4_MESH)
n = g.n
v = np.arange(n); cube = v // 6
x, y, z = cube // (N * N), (cube // N) % N, cube % N
def blocked_index(B=8):
    bx, by, bz = x // B, y // B, z // B
    nb = (N + B - 1) // B
    return ((bx * nb + by) * nb + bz) * (B ** 3 * 6) + ((x % B) * B + (y % B)) * B * 6 + (z % B) * 6 + v % 6
rand = prio(n).astype(np.int32); ident = v.astype(np.int32)
cases = {
    "lex ranges 2048": v // 2048,
    "blocked8 ranges 2048": np.argsort(np.argsort(blocked_index())) // 2048,
    "box 7x7x7": (x // 7) * 10000 + (y // 7) * 100 + z // 7,
    "box 4x4x21": (x // 4) * 10000 + (y // 4) * 100 + z // 21,
    "box 10x3x11": (x // 10) * 10000 + (y // 3) * 100 + z // 11,
    "box 14x14x14 (8x)": (x // 14) * 10000 + (y // 14) * 100 + z // 14,
}
sel = os.environ.get("SIM_CASES")
for name, t in cases.items():
    if sel and not any(k in name for k in sel.split(",")):
        continue
    for pname, pr, hp in [(a, b, c) for (a, b, c) in (("rand", rand, 0), ("rand+heap", rand, 1), ("ident", ident, 0), ("rand+gs", rand, 2), ("ident+gs", ident, 2)) if a in os.environ.get("SIM_PRIO", "rand,ident").split(",")]:
        t0 = time.time(); o = sim(g, t, pr, hp & 1, hp >> 1)
        print(f"{name:22s} {pname:9s} passes={o[0]:4d} visits={o[1]:7d} visited/n={o[2]/n:6.1f} raises/n={o[3]/n:6.2f}  ({time.time()-t0:.1f}s)", flush=True)
