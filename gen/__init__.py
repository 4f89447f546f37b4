"""Seeded synthetic input generators (shared by tests, bench and the oracle runs).

Holds none of the SCC method's arithmetic -- only graph construction.  The C++ core
(graphgen.cpp) uses counter-based hashing, so every graph is bit-reproducible.

Config recipes follow BASELINE.json ``configs`` and SURVEY.md Sec. 8(d):

* ``c1``  tiny: the worked example (tests/golden/appendix_a.json) and G(n=2000, m=8000), seed 1
* ``c2``  Kuhn-6 tet mesh sweep graph, N=55 -> n = 998,250, kappa=0.06, ordinate 0, seed 2
* ``c3``  R-MAT scale 22, edge factor 16, (a,b,c)=(.57,.19,.19), relabelled, seed 3
* ``c4``  tet mesh N=140 -> n = 16,464,000, kappa 0.05 with 0.25 hot spots in 1/10 of
          8^3-cube blocks, ordinate 0, seed 4
* ``c5``  64 meshes N=70 (n = 2,058,000 each), one per ordinate d, seed 5+d, as c4 otherwise
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "graphgen.cpp")
_LIB = os.path.join(_HERE, "libgraphgen.so")
_lib = None

ORDERS = {"lex": 0, "blocked8": 1}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-ffp-contract=off",
                               "-fno-fast-math", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i32p = ctypes.POINTER(ctypes.c_int32)
        dp = ctypes.POINTER(ctypes.c_double)
        lib.gen_mesh.restype = ctypes.c_int64
        lib.gen_mesh.argtypes = [ctypes.c_int64, ctypes.c_int, dp, ctypes.c_double, ctypes.c_double,
                                 ctypes.c_int, ctypes.c_int, ctypes.c_uint64, i32p, i32p]
        lib.gen_rmat.restype = ctypes.c_int64
        lib.gen_rmat.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                 ctypes.c_double, ctypes.c_uint64, ctypes.c_int, i32p, i32p]
        lib.gen_gnm.restype = ctypes.c_int64
        lib.gen_gnm.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_uint64, i32p, i32p]
        lib.csr_hash.restype = ctypes.c_uint64
        lib.csr_hash.argtypes = [ctypes.c_int64, i32p, ctypes.c_int64, i32p]
        _lib = lib
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))


@dataclass
class Graph:
    """CSR with int32 offsets and column indices (host, numpy)."""
    row_ptr: np.ndarray
    col_idx: np.ndarray
    name: str = ""

    @property
    def n(self) -> int:
        return int(self.row_ptr.shape[0] - 1)

    @property
    def nnz(self) -> int:
        return int(self.col_idx.shape[0])

    def hash(self) -> int:
        return int(_load().csr_hash(self.n, _p(self.row_ptr), self.nnz, _p(self.col_idx)))


# ---------------------------------------------------------------- ordinates
# 2 hemispheres x 4 Gauss-Legendre polar levels x 8 azimuths offset by pi/8
# the four positive Gauss-Legendre nodes (8-point rule), ordered so that d = 0 is the most
# oblique direction (all |Omega_i - Omega_j| large), the generic case for sweep graphs
_GL_POS = [0.7966664774136267, 0.5255324099163290, 0.9602898564975363, 0.1834346424956498]


def ordinate(d: int) -> tuple[float, float, float]:
    """Discrete ordinate d in [0, 64): hemisphere = d // 32, polar level = (d // 8) % 4,
    azimuth = d % 8 at phi = pi/8 + j*pi/4.  Unit vector (x, y, z)."""
    if not 0 <= d < 64:
        raise ValueError("ordinate index must be in [0, 64)")
    hemi, lvl, j = d // 32, (d // 8) % 4, d % 8
    mu = _GL_POS[lvl] * (1.0 if hemi == 0 else -1.0)
    phi = math.pi / 8 + j * math.pi / 4
    s = math.sqrt(1.0 - mu * mu)
    return (s * math.cos(phi), s * math.sin(phi), mu)


# ---------------------------------------------------------------- generators
def mesh(N: int, omega=None, kappa: float = 0.06, kappa_hot: float = 0.0, hot_mod: int = 0,
         Q: int = 4, seed: int = 2, order: str = "lex") -> Graph:
    """Directed sweep graph of a Kuhn-6 tet mesh of an N^3 cube grid."""
    if omega is None:
        omega = ordinate(0)
    n = 6 * N ** 3
    rp = np.empty(n + 1, dtype=np.int32)
    ci = np.empty(4 * n, dtype=np.int32)
    om = (ctypes.c_double * 3)(*omega)
    nnz = _load().gen_mesh(N, ORDERS[order], om, kappa, kappa_hot, hot_mod, Q, seed, _p(rp), _p(ci))
    return Graph(rp, ci[:nnz].copy(), f"mesh N={N} {order}")


def rmat(scale: int, edge_factor: int = 16, a: float = 0.57, b: float = 0.19, c: float = 0.19,
         seed: int = 3, permute: bool = True) -> Graph:
    n = 1 << scale
    rp = np.empty(n + 1, dtype=np.int32)
    ci = np.empty(edge_factor * n, dtype=np.int32)
    nnz = _load().gen_rmat(scale, edge_factor, a, b, c, seed, int(permute), _p(rp), _p(ci))
    return Graph(rp, ci[:nnz].copy(), f"rmat scale={scale}")


def gnm(n: int, m: int, seed: int = 1) -> Graph:
    rp = np.empty(n + 1, dtype=np.int32)
    ci = np.empty(max(m, 1), dtype=np.int32)
    nnz = _load().gen_gnm(n, m, seed, _p(rp), _p(ci))
    return Graph(rp, ci[:nnz].copy(), f"gnm n={n} m={m}")


def from_edges(n: int, edges, name: str = "") -> Graph:
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    if e.size:
        e = e[np.lexsort((e[:, 1], e[:, 0]))]
    counts = np.bincount(e[:, 0], minlength=n) if e.size else np.zeros(n, dtype=np.int64)
    rp = np.zeros(n + 1, dtype=np.int32)
    np.cumsum(counts, out=rp[1:])
    ci = e[:, 1].astype(np.int32) if e.size else np.zeros(0, dtype=np.int32)
    return Graph(rp, ci, name)


def appendix_a() -> Graph:
    import json
    p = os.path.join(os.path.dirname(_HERE), "tests", "golden", "appendix_a.json")
    g = json.load(open(p))
    return from_edges(g["n"], g["edges"], "appendix A")


# ---------------------------------------------------------------- BASELINE.json configs
C4_MESH = dict(kappa=0.05, kappa_hot=0.25, hot_mod=10, Q=4)


def config(name: str, order: str = "lex", d: int = 0, scale: int | None = None):
    """Return the Graph (or list of Graphs for c5) of a BASELINE.json config."""
    if name == "c1":
        return gnm(2000, 8000, seed=1)
    if name == "c2":
        return mesh(55, ordinate(0), kappa=0.06, seed=2, order=order)
    if name == "c3":
        return rmat(22 if scale is None else scale, 16, seed=3)
    if name == "c4":
        return mesh(140, ordinate(0), seed=4, order=order, **C4_MESH)
    if name == "c5":
        return [mesh(70, ordinate(k), seed=5 + k, order=order, **C4_MESH) for k in range(64)]
    if name == "c5one":   # one graph of the c5 batch
        return mesh(70, ordinate(d), seed=5 + d, order=order, **C4_MESH)
    raise ValueError(name)
