"""CPU oracle for the ECL-SCC hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product package
``paper_conf_sc_alabandisbb23_b200`` never imports it, and it never imports the product:
the two share no code.  The only thing both sides see is the generated CSR from ``gen/``.

Functions (each cites the passage it follows; P:n = /root/reference/PAPER.md line n):

* ``tarjan_labels(row_ptr, col_idx)`` -- O1: SCCs by Tarjan's algorithm (P:53, P:79,
  P:208), each labelled by its largest vertex ID.  The plain definition.
* ``ecl_scc(row_ptr, col_idx, reset_all=False, compress=False, trim=False, snap_iter=0,
  trim2=False, four=False, raise_=False)`` -- O2: Alg. 1 in the paper's order
  with Jacobi Phase-2 rounds and the per-iteration trace.  Flags follow the readings in
  DESIGN.md: R1/R2, path compression, Trim-1 and Trim-2, the 4-signature
  variant, the sound variant of the P:190 trick.
* ``scc_levels(row_ptr, col_idx, labels)`` -- O4: the sweep levels of the SCC condensation
  (Table 2's "DAG depth"): Kahn's algorithm on the condensation, level = longest path
  from a source SCC.  Returns (levels per vertex, depth).

Both live in ``oracle.c`` and run single-threaded.  Pins: tests/test_oracle.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

RESET_ALL = 1
COMPRESS = 2
TRIM = 4
TRIM2 = 8
FOUR = 16
RAISE = 32

_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so (gcc -O2; no -ffast-math, integer-only code)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i32p = ctypes.POINTER(ctypes.c_int32)
        i64p = ctypes.POINTER(ctypes.c_int64)
        lib.oracle_tarjan_labels.restype = ctypes.c_int64
        lib.oracle_tarjan_labels.argtypes = [ctypes.c_int32, i64p, i32p, i32p]
        lib.oracle_ecl_scc.restype = ctypes.c_int32
        lib.oracle_ecl_scc.argtypes = [ctypes.c_int32, i64p, i32p, ctypes.c_uint32, i32p,
                                       ctypes.c_int32, i64p, i64p, i64p,
                                       ctypes.c_int32, i32p, i32p]
        lib.oracle_scc_levels.restype = ctypes.c_int32
        lib.oracle_scc_levels.argtypes = [ctypes.c_int32, i64p, i32p, i32p, i32p]
        _lib = lib
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def _csr(row_ptr, col_idx):
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    n = rp.shape[0] - 1
    if n < 0 or rp[0] != 0 or rp[-1] != ci.shape[0]:
        raise ValueError("malformed CSR")
    if ci.size and (ci.min() < 0 or ci.max() >= n):
        raise ValueError("column index out of range")
    return n, rp, ci


def tarjan_labels(row_ptr, col_idx) -> np.ndarray:
    """O1: labels[v] = max vertex ID of v's SCC (Tarjan + max relabel)."""
    n, rp, ci = _csr(row_ptr, col_idx)
    labels = np.empty(n, dtype=np.int32)
    if n == 0:
        return labels
    r = _load().oracle_tarjan_labels(n, _p(rp, ctypes.c_int64), _p(ci, ctypes.c_int32),
                                     _p(labels, ctypes.c_int32))
    if r < 0:
        raise MemoryError("oracle_tarjan_labels")
    return labels


def scc_levels(row_ptr, col_idx, labels) -> tuple[np.ndarray, int]:
    """O4: (level of each vertex's SCC in the condensation DAG, depth = max level + 1)."""
    n, rp, ci = _csr(row_ptr, col_idx)
    lab = np.ascontiguousarray(labels, dtype=np.int32)
    levels = np.empty(n, dtype=np.int32)
    if n == 0:
        return levels, 0
    d = _load().oracle_scc_levels(n, _p(rp, ctypes.c_int64), _p(ci, ctypes.c_int32),
                                  _p(lab, ctypes.c_int32), _p(levels, ctypes.c_int32))
    if d == -1:
        raise MemoryError("oracle_scc_levels")
    if d == -2:
        raise ValueError("labels do not induce an acyclic condensation")
    return levels, int(d)


@dataclass
class Trace:
    labels: np.ndarray
    iterations: int
    edges_in: list = field(default_factory=list)
    passes: list = field(default_factory=list)
    edges_kept: list = field(default_factory=list)
    snap_in: np.ndarray | None = None
    snap_out: np.ndarray | None = None


def ecl_scc(row_ptr, col_idx, reset_all: bool = False, compress: bool = False,
            trim: bool = False, snap_iter: int = 0, max_trace: int = 4096, trim2: bool = False,
            four: bool = False, raise_: bool = False) -> Trace:
    """O2: literal Alg. 1 with Jacobi Phase 2; returns labels and the per-iteration trace.
    trim2: Trim-2; four: the 4-signature variant; raise_: the sound variant of
    the P:190 trick."""
    n, rp, ci = _csr(row_ptr, col_idx)
    flags = ((RESET_ALL if reset_all else 0) | (COMPRESS if compress else 0) | (TRIM if trim else 0)
             | (TRIM2 if trim2 else 0) | (FOUR if four else 0) | (RAISE if raise_ else 0))
    labels = np.empty(n, dtype=np.int32)
    ein = np.zeros(max_trace, dtype=np.int64)
    pas = np.zeros(max_trace, dtype=np.int64)
    kept = np.zeros(max_trace, dtype=np.int64)
    sin = np.zeros(max(n, 1), dtype=np.int32)
    sout = np.zeros(max(n, 1), dtype=np.int32)
    if n == 0:
        return Trace(labels, 0)
    it = _load().oracle_ecl_scc(n, _p(rp, ctypes.c_int64), _p(ci, ctypes.c_int32), flags,
                                _p(labels, ctypes.c_int32), max_trace,
                                _p(ein, ctypes.c_int64), _p(pas, ctypes.c_int64),
                                _p(kept, ctypes.c_int64), snap_iter,
                                _p(sin, ctypes.c_int32), _p(sout, ctypes.c_int32))
    if it == -1:
        raise MemoryError("oracle_ecl_scc")
    if it == -2:
        raise RuntimeError("oracle_ecl_scc: iteration cap reached (non-terminating rule mix?)")
    if it == -3:
        raise ValueError("oracle_ecl_scc: Trim-2 needs rule R2 (reset_all=False)")
    k = min(it, max_trace)
    tr = Trace(labels, it, ein[:k].tolist(), pas[:k].tolist(), kept[:k].tolist())
    if 1 <= snap_iter <= it:
        tr.snap_in, tr.snap_out = sin[:n].copy(), sout[:n].copy()
    return tr


def csr_from_edges(n: int, edges) -> tuple[np.ndarray, np.ndarray]:
    """Edge list -> CSR (rows in source order, each row sorted).  Test convenience."""
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    order = np.lexsort((e[:, 1], e[:, 0])) if e.size else np.zeros(0, dtype=np.int64)
    e = e[order]
    counts = np.bincount(e[:, 0], minlength=n) if e.size else np.zeros(n, dtype=np.int64)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return rp, e[:, 1].astype(np.int32) if e.size else np.zeros(0, dtype=np.int32)
