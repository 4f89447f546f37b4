"""The C-ABI library loads and exports every symbol include/ecl_scc.h declares; host-only
entry points and argument validation (no GPU compute), -m "not gpu"."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_sc_alabandisbb23_b200 as E

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "ecl_scc.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ecl_scc\w*)\s*\(", src)))


def test_library_exports_every_header_symbol():
    L = E.lib()
    names = header_functions()
    assert len(names) >= 15
    for name in names:
        assert hasattr(L, name), name
    assert set(names) == set(E.ABI_SYMBOLS)


def test_version_and_status_strings():
    assert E.lib().ecl_scc_version() == 100
    for s in range(7):
        assert E.status_string(s)
    assert E.status_string(0) == "ok"


def test_argument_errors_without_gpu():
    L = E.lib()
    assert L.ecl_scc(-1, 0, None, None, None) == E.EINVAL
    assert L.ecl_scc(3, -1, None, None, None) == E.EINVAL
    assert L.ecl_scc(3, 0, None, None, None) == E.EINVAL          # NULL row_ptr with n > 0
    assert b"NULL" in L.ecl_scc_last_error()
    assert L.ecl_scc(0, 0, None, None, None) == E.OK               # n == 0 -> nothing to do
    assert L.ecl_scc(10, 1 << 31, ctypes.c_void_p(16), ctypes.c_void_p(16), ctypes.c_void_p(16)) == E.EUNSUPPORTED
    assert L.ecl_scc_plan_create(-1, 0, 0, None) == E.EINVAL
    assert L.ecl_scc_batched(-1, None, None, None, None, None, None, None, None) == E.EINVAL
    assert L.ecl_scc_batched_host(-1, None, None, None, None, None, None, None, None) == E.EINVAL
    assert L.ecl_scc_batched_host(0, None, None, None, None, None, None, None, None) == E.OK


def test_partition_rows_balanced():
    rng = np.random.default_rng(0)
    deg = rng.integers(0, 50, 10000)
    rp = np.zeros(10001, dtype=np.int32)
    np.cumsum(deg, out=rp[1:])
    for P in (1, 2, 3, 8):
        b = E.ecl_scc_partition_rows(P, rp)
        assert b[0] == 0 and b[-1] == 10000 and all(b[i] <= b[i + 1] for i in range(P))
        load = [rp[b[i + 1]] - rp[b[i]] for i in range(P)]
        assert max(load) - min(load) <= 2 * 50 + 1


def test_levels_and_host_argument_errors_without_gpu():
    L = E.lib()
    p = ctypes.c_void_p(16)
    depth = ctypes.c_int32(7)
    assert L.ecl_scc_levels(-1, 0, None, None, None, None, None, None, None) == E.EINVAL
    assert L.ecl_scc_levels(3, 0, p, None, None, p, None, None, None) == E.EINVAL     # NULL labels
    assert L.ecl_scc_levels(0, 0, None, None, None, None, ctypes.byref(depth), None, None) == E.OK
    assert depth.value == 0                                                          # empty graph
    assert L.ecl_scc_host(-1, 0, None, None, None, None, None, None) == E.EINVAL
    assert L.ecl_scc_host(3, 2, p, None, p, None, None, None) == E.EINVAL             # NULL col_idx
    assert L.ecl_scc_host(0, 0, None, None, None, None, None, None) == E.OK
