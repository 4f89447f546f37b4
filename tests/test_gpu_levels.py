"""GPU parity of the sweep levels (ecl_scc_levels, levels.cuh) against oracle O4.

Levels are integers with a unique definition (longest condensation path ending in a vertex's
SCC; Table 2's "DAG depth"), so every comparison is bit-exact.  The labels fed in are
the GPU's own ecl_scc output, checked against Tarjan first.
"""
import random

import numpy as np
import pytest
import torch

import gen
import oracle
import paper_conf_sc_alabandisbb23_b200 as E

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def check(g, plan=None):
    """Both level algorithms against O4: the default (Kahn's rule per tile on the tile queue
    where the cross edges mostly stay inside tiles, else Kahn's global rounds) and Kahn's
    global rounds alone (a plan with ECL_SCC_NO_ASYNC)."""
    rp, ci = dev(g.row_ptr), dev(g.col_idx)
    lab = E.ecl_scc(rp, ci, plan=plan)
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    np.testing.assert_array_equal(lab.cpu().numpy(), truth)
    exp, edepth = oracle.scc_levels(g.row_ptr, g.col_idx, truth)
    rounds = E.Plan(max(g.n, 1), max(g.nnz, 1), E.NO_ASYNC)
    for p in (plan, rounds):
        lv, depth = E.ecl_scc_levels(rp, ci, lab, plan=p)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(lv.cpu().numpy(), exp)
        assert depth == edepth
    return depth


def test_levels_random_small():
    rng = random.Random(21)
    for trial in range(120):
        n = rng.randrange(1, 400)
        m = rng.randrange(0, 3 * n)
        g = gen.from_edges(n, [(rng.randrange(n), rng.randrange(n)) for _ in range(m)])
        check(g)


def test_levels_closed_forms():
    n = 100_000
    perm = np.random.default_rng(2).permutation(n)
    assert check(gen.from_edges(n, np.stack([perm[:-1], perm[1:]], 1))) == n       # a path: depth n
    assert check(gen.from_edges(n, np.stack([perm, np.roll(perm, -1)], 1))) == 1    # one cycle
    assert check(gen.from_edges(50, [])) == 1                                     # no edges
    k = 5                                                                         # chain of k-cycles
    e = [(k * j + i, k * j + (i + 1) % k) for j in range(300) for i in range(k)] + \
        [(k * j + k - 1, k * (j + 1)) for j in range(299)]
    assert check(gen.from_edges(1500, e)) == 300


def test_levels_meshes_and_rmat():
    for g in (gen.config("c1"), gen.config("c2", order="lex"), gen.config("c2", order="blocked8"),
              gen.mesh(40, gen.ordinate(3), seed=8, order="blocked8", **gen.C4_MESH), gen.config("c3")):
        check(g)


def test_levels_c4_with_plan():
    g = gen.config("c4", order="blocked8")
    plan = E.Plan(g.n, g.nnz)
    assert check(g, plan) > 100                    # a deep DAG (the SCCs form a deep DAG)


def test_levels_reject_bad_labels():
    g = gen.from_edges(4, [(0, 1), (1, 0), (2, 3)])
    rp, ci = dev(g.row_ptr), dev(g.col_idx)
    with pytest.raises(E.EclSccError) as ex:                  # 0 and 1 apart: cyclic condensation
        E.ecl_scc_levels(rp, ci, dev([0, 1, 2, 3]))
    assert ex.value.status == E.ERANGE
    with pytest.raises(E.EclSccError) as ex:                  # a label outside [0, n)
        E.ecl_scc_levels(rp, ci, dev([1, 1, 2, 9]))
    assert ex.value.status == E.ERANGE
    # far out of range on a large graph (would index far outside every workspace array):
    # rejected before any label-indexed kernel runs, and the context stays usable
    n = 200_000
    g = gen.from_edges(n, np.stack([np.arange(n - 1), np.arange(1, n)], 1))
    rp, ci = dev(g.row_ptr), dev(g.col_idx)
    for bad in (2**31 - 2, -5):
        lab = np.arange(n, dtype=np.int32)
        lab[[3, n // 2, n - 1]] = bad
        with pytest.raises(E.EclSccError) as ex:
            E.ecl_scc_levels(rp, ci, dev(lab))
        assert ex.value.status == E.ERANGE
    lv, depth = E.ecl_scc_levels(rp, ci, dev(np.arange(n, dtype=np.int32)))
    assert depth == n and (lv.cpu().numpy() == np.arange(n)).all()


@pytest.mark.parametrize("flags", [0, E.NO_ASYNC])
def test_levels_cyclic_labels_on_a_mesh(flags):
    """Labels that split SCCs make the condensation cyclic: both algorithms report ERANGE
    (tile mode: nodes left unprocessed at the queue's fixed point), and the context stays
    usable."""
    g = gen.config("c2", order="blocked8")
    rp, ci = dev(g.row_ptr), dev(g.col_idx)
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    assert (truth != np.arange(g.n)).any()                      # the mesh has non-trivial SCCs
    plan = E.Plan(g.n, g.nnz, flags)
    with pytest.raises(E.EclSccError) as ex:
        E.ecl_scc_levels(rp, ci, dev(np.arange(g.n, dtype=np.int32)), plan=plan)
    assert ex.value.status == E.ERANGE
    lv, depth = E.ecl_scc_levels(rp, ci, dev(truth), plan=plan)
    exp, edepth = oracle.scc_levels(g.row_ptr, g.col_idx, truth)
    np.testing.assert_array_equal(lv.cpu().numpy(), exp)
    assert depth == edepth
