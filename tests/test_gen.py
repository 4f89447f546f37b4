"""Synthetic input generators (gen/): structure and reproducibility, -m "not gpu"."""
import numpy as np

import gen
import oracle


def _pairs(g):
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    return src, g.col_idx


def test_mesh_structure_and_dag_at_zero_curvature():
    for order in ("lex", "blocked8"):
        for N in (3, 9, 12):
            g = gen.mesh(N, gen.ordinate(0), kappa=0.0, seed=1, order=order)
            assert g.n == 6 * N ** 3
            src, dst = _pairs(g)
            assert (src != dst).all()
            und = np.unique(np.minimum(src, dst).astype(np.int64) * g.n + np.maximum(src, dst))
            faces = 6 * N ** 3 + 6 * N ** 2 * (N - 1)      # interior faces of the Kuhn mesh
            assert und.size == faces
            assert g.nnz == faces                          # flat faces: exactly one direction
            assert np.diff(g.row_ptr).max() <= 4
            # linear (flat) elements are convex -> every SCC is trivial
            np.testing.assert_array_equal(oracle.tarjan_labels(g.row_ptr, g.col_idx), np.arange(g.n))


def test_mesh_curved_faces_make_cycles():
    g = gen.mesh(10, gen.ordinate(0), kappa=0.3, seed=3)
    lab = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    assert (lab != np.arange(g.n)).sum() > 0
    src, dst = _pairs(g)
    und = np.unique(np.minimum(src, dst).astype(np.int64) * g.n + np.maximum(src, dst))
    assert und.size == 6 * 10 ** 3 + 6 * 10 ** 2 * 9    # same faces, some doubled
    assert g.nnz > und.size


def test_orders_are_permutations_of_each_other():
    """lex and blocked8 number the same elements differently: same degree multiset and
    same SCC size multiset at kappa=0 (flat faces need no RNG)."""
    a = gen.mesh(11, gen.ordinate(5), kappa=0.0, order="lex")
    b = gen.mesh(11, gen.ordinate(5), kappa=0.0, order="blocked8")
    assert a.nnz == b.nnz
    np.testing.assert_array_equal(np.sort(np.diff(a.row_ptr)), np.sort(np.diff(b.row_ptr)))


def test_reproducible_hashes():
    g1 = gen.mesh(8, gen.ordinate(3), kappa=0.1, seed=9)
    g2 = gen.mesh(8, gen.ordinate(3), kappa=0.1, seed=9)
    assert g1.hash() == g2.hash()
    assert gen.mesh(8, gen.ordinate(3), kappa=0.1, seed=10).hash() != g1.hash()
    r1, r2 = gen.rmat(12, seed=3), gen.rmat(12, seed=3)
    assert r1.hash() == r2.hash()


def test_rmat_and_gnm():
    r = gen.rmat(14, 16, seed=3)
    assert r.n == 1 << 14
    src, dst = _pairs(r)
    assert (src != dst).all()
    key = src.astype(np.int64) * r.n + dst
    assert (np.diff(key) > 0).all()                       # sorted rows, no duplicates
    assert 0.8 * 16 * r.n < r.nnz <= 16 * r.n
    deg = np.diff(r.row_ptr)
    assert deg.max() > 20 * deg.mean()                    # power-law-like skew
    g = gen.gnm(2000, 8000, seed=1)
    assert g.nnz == 8000
    src, dst = _pairs(g)
    key = src.astype(np.int64) * g.n + dst
    assert (src != dst).all() and np.unique(key).size == 8000


def test_ordinates_unit_and_distinct():
    om = np.array([gen.ordinate(d) for d in range(64)])
    np.testing.assert_allclose(np.linalg.norm(om, axis=1), 1.0)
    assert np.unique(np.round(om, 12), axis=0).shape[0] == 64
