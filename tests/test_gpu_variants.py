"""GPU parity of the paper's variants against oracle O2 with the same flags:
Trim-2 (ECL_SCC_TRIM2) and the 4-signature method (ECL_SCC_FOUR_SIG).

Labels are compared bit-exactly with Tarjan; the per-iteration trace (live edges entering
Phase 2, kept edges, signatures after every Phase 2) with O2 run with the same variant
flags on the same graph (relabelled by the GPU's priorities pi, reading 16).
"""
import random

import numpy as np
import pytest
import torch

import gen
import oracle
import paper_conf_sc_alabandisbb23_b200 as E
from prio_ref import prio

pytestmark = pytest.mark.gpu

VARIANTS = {"trim2": (E.TRIM2, dict(trim2=True)),
            "four": (E.FOUR_SIG, dict(four=True)),
            "trim2+four": (E.TRIM2 | E.FOUR_SIG, dict(trim2=True, four=True))}


def dev(g):
    return torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda()


def relabel(g, pi):
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    return gen.from_edges(g.n, np.stack([pi[src], pi[g.col_idx]], 1))


def run(g, flags):
    rp, ci = dev(g)
    lab, st = E.ecl_scc(rp, ci, plan=E.Plan(g.n, g.nnz, flags), stats=True)
    torch.cuda.synchronize()
    return lab.cpu().numpy(), st


def check(g, flags, okw, snaps=True, max_iters=None):
    lab, st = run(g, flags)
    np.testing.assert_array_equal(lab, oracle.tarjan_labels(g.row_ptr, g.col_idx))
    ids = bool(flags & E.IDENTITY_IDS)
    trim = not (flags & E.NO_TRIM)
    pi = np.arange(g.n) if ids else prio(g.n)
    og = g if ids else relabel(g, pi)
    tr = oracle.ecl_scc(og.row_ptr, og.col_idx, trim=trim, **okw)
    k = tr.iterations
    assert st["iterations"] == k
    assert st["edges_in"] == tr.edges_in[:64]
    assert st["edges_kept"] == tr.edges_kept[:max(min(k, 64) - 1, 0)]
    if snaps:
        rp, ci = dev(g)
        for it in range(1, (k if max_iters is None else min(k, max_iters)) + 1):
            s = oracle.ecl_scc(og.row_ptr, og.col_idx, trim=trim, snap_iter=it, **okw)
            gi, go, _ = E.ecl_scc_debug_run(rp, ci, it, flags=flags)
            np.testing.assert_array_equal(gi.cpu().numpy(), s.snap_in[pi], err_msg=f"in, iteration {it}")
            np.testing.assert_array_equal(go.cpu().numpy(), s.snap_out[pi], err_msg=f"out, iteration {it}")
    return st


@pytest.mark.parametrize("name", sorted(VARIANTS))
def test_variants_random_small(name):
    fl, okw = VARIANTS[name]
    rng = random.Random(hash(name) & 0xFFFF)
    for trial in range(80):
        n = rng.randrange(1, 300)
        edges = [(rng.randrange(n), rng.randrange(n)) for _ in range(rng.randrange(0, 3 * n))]
        for _ in range(rng.randrange(0, 6)):                    # planted 2-cycles
            a, b = rng.randrange(n), rng.randrange(n)
            edges += [(a, b), (b, a)]
        g = gen.from_edges(n, edges)
        for extra in (0, E.IDENTITY_IDS, E.NO_ASYNC, E.SYNC_PASSES, E.FORCE_REORDER):
            check(g, fl | extra, okw, snaps=trial % 8 == 0)
        if "trim2" not in name:
            check(g, fl | E.NO_TRIM, okw, snaps=trial % 8 == 0)


@pytest.mark.parametrize("name", sorted(VARIANTS))
def test_variants_c1_and_meshes(name):
    fl, okw = VARIANTS[name]
    check(gen.config("c1"), fl, okw)
    check(gen.appendix_a(), fl | E.IDENTITY_IDS, okw)
    g = gen.mesh(24, gen.ordinate(9), seed=4, order="blocked8", **gen.C4_MESH)   # 82,944 vertices
    check(g, fl, okw, max_iters=4)


@pytest.mark.parametrize("name", sorted(VARIANTS))
def test_variants_long_rows(name):
    """Power-law rows (> 64 entries, chunk kernels and the warp paths of the compaction)."""
    fl, okw = VARIANTS[name]
    rng = np.random.default_rng(11)
    n = 20_000
    src = np.concatenate([np.full(3000, 17), rng.integers(0, n, 40_000), np.arange(0, 2000, 2)])
    dst = np.concatenate([rng.integers(0, n, 3000), rng.integers(0, n, 40_000), np.arange(1, 2001, 2)])
    src = np.concatenate([src, np.arange(1, 2001, 2)])          # 1000 bidirectional pairs
    dst = np.concatenate([dst, np.arange(0, 2000, 2)])
    check(gen.from_edges(n, np.stack([src, dst], 1)), fl, okw, max_iters=3)
    check(gen.rmat(14, 16, seed=7), fl, okw, snaps=False)


def test_variant_flag_errors():
    with pytest.raises(E.EclSccError) as ex:
        E.Plan(10, 10, E.TRIM2 | E.NO_TRIM)
    assert ex.value.status == E.EINVAL


def test_variants_c2_full_trace():
    g = gen.config("c2", order="blocked8")
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    og = relabel(g, prio(g.n))
    for name, (fl, okw) in VARIANTS.items():
        lab, st = run(g, fl)
        np.testing.assert_array_equal(lab, truth, err_msg=name)
        tr = oracle.ecl_scc(og.row_ptr, og.col_idx, trim=True, **okw)
        assert st["iterations"] == tr.iterations and st["edges_in"] == tr.edges_in[:64], name


# ----------------------------------------------------------------- f2: compression and the P:190 variant
TRICKS = {"compress": E.COMPRESS, "raise": E.RAISE, "compress+raise": E.COMPRESS | E.RAISE}


@pytest.mark.parametrize("name", sorted(TRICKS))
def test_pass_count_variants_keep_the_trace(name):
    """Path compression and the sound P:190 variant change how values travel, never
    where Phase 2 ends (reading 12): labels, live / kept edges and every signature snapshot
    equal O2's plain trace (O2's own compress / raise_ flags give the same trace, pinned in
    tests/test_oracle.py)."""
    fl = TRICKS[name]
    rng = random.Random(len(name))
    for trial in range(60):
        n = rng.randrange(1, 300)
        edges = [(rng.randrange(n), rng.randrange(n)) for _ in range(rng.randrange(0, 3 * n))]
        g = gen.from_edges(n, edges)
        for extra in (0, E.IDENTITY_IDS, E.NO_ASYNC, E.NO_TRIM):
            check(g, fl | extra, {}, snaps=trial % 6 == 0)
    for g in (gen.config("c1"), gen.mesh(24, gen.ordinate(9), seed=4, order="blocked8", **gen.C4_MESH)):
        check(g, fl, {}, max_iters=4)
    perm = np.random.default_rng(2).permutation(200_000)                # one long cycle
    g = gen.from_edges(200_000, np.stack([perm, np.roll(perm, -1)], 1))
    lab, st = run(g, fl)
    assert (lab == 199_999).all()


def test_pass_count_variant_flag_errors():
    with pytest.raises(E.EclSccError) as ex:
        E.Plan(10, 10, E.COMPRESS | E.FOUR_SIG)
    assert ex.value.status == E.EINVAL


# ----------------------------------------------------------------- f2: thread-block-cluster pair tiles
def test_cluster_pair_tiles_keep_the_trace():
    """ECL_SCC_CLUSTER: two CTAs share one 4096-vertex block-local fixed point through DSMEM
    (csrc/cluster.cuh).  Only the schedule changes (reading 12): labels bit-exact, live / kept
    edges and every signature snapshot equal O2's trace -- on graphs spanning many pair tiles,
    so that both halves and the remote (DSMEM) slots are exercised."""
    rng = random.Random(4096)
    for trial in range(30):
        n = rng.randrange(1, 12_000) if trial % 3 else rng.randrange(1, 300)
        k = rng.randrange(0, 3 * n)
        src = np.array([rng.randrange(n) for _ in range(k)], dtype=np.int64)
        # mostly local edges (so pair tiles hold real intra- and cross-half work)
        dst = np.clip(src + np.array([rng.randrange(-3000, 3000) for _ in range(k)], dtype=np.int64), 0, n - 1)
        g = gen.from_edges(n, np.stack([src, dst], 1) if k else [])
        for extra in (0, E.IDENTITY_IDS, E.NO_TRIM):
            check(g, E.CLUSTER | extra, {}, snaps=trial % 5 == 0, max_iters=3)
    for g in (gen.config("c1"), gen.mesh(24, gen.ordinate(9), seed=4, order="blocked8", **gen.C4_MESH),
              gen.mesh(20, gen.ordinate(30), seed=8, order="lex", **gen.C4_MESH)):
        check(g, E.CLUSTER, {}, max_iters=4)
    check(gen.mesh(16, gen.ordinate(2), seed=3, **gen.C4_MESH), E.CLUSTER | E.FOUR_SIG, dict(four=True), max_iters=2)
    g = gen.config("c2", order="blocked8")
    lab, st = run(g, E.CLUSTER)
    np.testing.assert_array_equal(lab, oracle.tarjan_labels(g.row_ptr, g.col_idx))


@pytest.mark.parametrize("flags", [0, E.NO_KW, E.NO_TRIM, E.NO_TRIM | E.NO_KW])
def test_keep_word_layout_keeps_the_trace(flags):
    """The small-degree compaction (one 4-byte keep word per vertex, rows of <= 8 entries:
    every mesh) and the general layout (ECL_SCC_NO_KW) against O2: labels, per-iteration
    trace and signature snapshots; and a graph with longer rows takes the general path."""
    for g in (gen.mesh(14, gen.ordinate(5), seed=9, order="blocked8", **gen.C4_MESH), gen.config("c1")):
        check(g, flags, {}, max_iters=3)
    lab, st = run(gen.config("c2", order="blocked8"), flags)
    lab2, st2 = run(gen.config("c2", order="blocked8"), flags ^ E.NO_KW)
    np.testing.assert_array_equal(lab, lab2)
    assert st["edges_in"] == st2["edges_in"] and st["edges_kept"] == st2["edges_kept"]
