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


def _lex_of_blocked(N):
    """blocked8 element ID -> lexicographic element ID (the generator's two numberings)."""
    B = 8
    lex_of = np.empty(6 * N ** 3, dtype=np.int64)
    for x in range(N):
        for y in range(N):
            for z in range(N):
                bx, by, bz = x // B, y // B, z // B
                bsx, bsy, bsz = min(B, N - bx * B), min(B, N - by * B), min(B, N - bz * B)
                off = (bx * B) * N * N + bsx * (by * B) * N + bsx * bsy * (bz * B)
                cb = off + ((x - bx * B) * bsy + (y - by * B)) * bsz + (z - bz * B)
                cl = (x * N + y) * N + z
                lex_of[6 * cb:6 * cb + 6] = 6 * cl + np.arange(6)
    return lex_of


def test_orders_are_exact_relabellings_with_curvature():
    """At kappa > 0 (random curved faces, hot spots) blocked8 is the lex graph with the
    vertices renamed: the sorted edge lists agree after mapping blocked8 IDs to lex IDs."""
    for N, d in ((9, 0), (17, 13)):        # N=17: partial 8^3 blocks at the boundary
        kw = dict(kappa=0.05, kappa_hot=0.4, hot_mod=3, seed=11)
        a = gen.mesh(N, gen.ordinate(d), order="lex", **kw)
        b = gen.mesh(N, gen.ordinate(d), order="blocked8", **kw)
        assert a.nnz == b.nnz
        lex_of = _lex_of_blocked(N)
        assert np.unique(lex_of).size == a.n
        sa, da = _pairs(a)
        sb, db = _pairs(b)
        ka = np.sort(sa.astype(np.int64) * a.n + da)
        kb = np.sort(lex_of[sb] * a.n + lex_of[db])
        np.testing.assert_array_equal(ka, kb)
        assert (oracle.tarjan_labels(a.row_ptr, a.col_idx) != np.arange(a.n)).any()   # cycles exist


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
