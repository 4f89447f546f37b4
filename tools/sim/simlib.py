import ctypes, os, sys
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import gen  # noqa
from prio_ref import prio  # noqa
L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libtilesim.so"))
L.tilesim.restype = ctypes.c_int64
P = lambda a: a.ctypes.data_as(ctypes.c_void_p)

def run(g, tile_of, pr, heap=0, gs=0, order=None, window=1):
    out = np.zeros(4, dtype=np.int64)
    nt = int(tile_of.max()) + 1
    L.tilesim(ctypes.c_int32(g.n), P(g.row_ptr), P(g.col_idx), P(tile_of), ctypes.c_int32(nt), P(pr), P(out),
              ctypes.c_int(heap), ctypes.c_int(gs), P(order) if order is not None else None, ctypes.c_int32(window),
              ctypes.c_int32(0))
    return out

def mesh_coords(N, n):
    v = np.arange(n); cube = v // 6
    return v, cube // (N * N), (cube // N) % N, cube % N

def blocked_tiles(N, g, TT=2048, B=8):
    v, x, y, z = mesh_coords(N, g.n)
    bx, by, bz = x // B, y // B, z // B; nb = (N + B - 1) // B
    bidx = ((bx * nb + by) * nb + bz) * (B ** 3 * 6) + ((x % B) * B + (y % B)) * B * 6 + (z % B) * 6 + v % 6
    return (np.argsort(np.argsort(bidx)) // TT).astype(np.int32)
