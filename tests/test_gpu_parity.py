"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Labels are integers with a unique definition, so every comparison is
bit-exact.  Per-iteration states (live edge counts, signatures after each Phase 2) are
schedule independent (reading 12) and compared exactly against O2 with the same
trim rule.  Pass counts are schedule dependent and never compared.
"""
import json
import os
import random

import numpy as np
import pytest
import torch

import gen
import oracle
import paper_conf_sc_alabandisbb23_b200 as E
from prio_ref import prio

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def dev(g):
    return (torch.from_numpy(np.ascontiguousarray(g.row_ptr, dtype=np.int32)).cuda(),
            torch.from_numpy(np.ascontiguousarray(g.col_idx, dtype=np.int32)).cuda())


def gpu_labels(g, flags=0, plan=None):
    rp, ci = dev(g)
    if flags and plan is None:
        plan = E.Plan(g.n, g.nnz, flags)
    lab, st = E.ecl_scc(rp, ci, plan=plan, stats=True)
    torch.cuda.synchronize()
    return lab.cpu().numpy(), st


def relabel(g, pi):
    """The same graph with vertex v renamed pi[v] (rows permuted accordingly)."""
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    return gen.from_edges(g.n, np.stack([pi[src], pi[g.col_idx]], 1))


def check_trace(g, trim, flags=0, max_iters=None):
    """GPU per-iteration edge counts and signatures == O2's (same trim rule).

    With raw IDs (IDENTITY_IDS) O2 runs on the graph itself.  By default the GPU
    propagates priorities pi(v) (reading 16), which is Alg. 1 on the graph
    relabelled by pi: O2 runs on that graph and vertex v is compared at pi(v)."""
    fl = flags | (0 if trim else E.NO_TRIM)
    ids = bool(fl & E.IDENTITY_IDS)
    pi = np.arange(g.n) if ids else prio(g.n)
    og = g if ids else relabel(g, pi)
    tr = oracle.ecl_scc(og.row_ptr, og.col_idx, trim=trim)
    rp, ci = dev(g)
    _, st = gpu_labels(g, fl)
    k = tr.iterations
    assert st["iterations"] == k
    assert st["edges_in"] == tr.edges_in[:64]
    assert st["edges_kept"] == tr.edges_kept[:max(min(k, 64) - 1, 0)]
    for it in range(1, (k if max_iters is None else min(k, max_iters)) + 1):
        s = oracle.ecl_scc(og.row_ptr, og.col_idx, trim=trim, snap_iter=it)
        gi, go, _ = E.ecl_scc_debug_run(rp, ci, it, flags=fl)
        np.testing.assert_array_equal(gi.cpu().numpy(), s.snap_in[pi], err_msg=f"in, iteration {it}")
        np.testing.assert_array_equal(go.cpu().numpy(), s.snap_out[pi], err_msg=f"out, iteration {it}")


# ----------------------------------------------------------------- C1: worked example
@pytest.mark.parametrize("flags", [0, E.SYNC_PASSES, E.NO_DIRTY])
def test_appendix_a(flags):
    """The hand-derived worked example (raw IDs, so the golden signatures apply as is)."""
    gold = json.load(open(os.path.join(GOLDEN, "appendix_a.json")))
    g = gen.appendix_a()
    for trim, key in ((False, "r2_no_trim"), (True, "r2_trim1")):
        fl = flags | E.IDENTITY_IDS | (0 if trim else E.NO_TRIM)
        lab, st = gpu_labels(g, fl)
        np.testing.assert_array_equal(lab, gold["labels"])
        exp = gold[key]
        assert st["edges_in"] == exp["edges_in"]
        assert st["edges_kept"] == exp["edges_kept"][:-1]
        rp, ci = dev(g)
        for it in range(1, len(exp["in"]) + 1):
            gi, go, _ = E.ecl_scc_debug_run(rp, ci, it, flags=fl)
            np.testing.assert_array_equal(gi.cpu().numpy(), exp["in"][it - 1])
            np.testing.assert_array_equal(go.cpu().numpy(), exp["out"][it - 1])


def test_random_small_graphs_labels_and_traces():
    rng = random.Random(77)
    for trial in range(150):
        n = rng.randrange(1, 300)
        m = rng.randrange(0, 4 * n)
        edges = [(rng.randrange(n), rng.randrange(n)) for _ in range(m)]
        g = gen.from_edges(n, edges)
        truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
        for flags in (0, E.NO_TRIM, E.IDENTITY_IDS, E.SYNC_PASSES, E.NO_DIRTY, E.FORCE_REORDER, E.NO_PACK,
                      E.NO_ASYNC):
            lab, _ = gpu_labels(g, flags)
            np.testing.assert_array_equal(lab, truth, err_msg=f"trial {trial} flags {flags}")
        if trial % 10 == 0:
            check_trace(g, trim=True)
            check_trace(g, trim=False)
            check_trace(g, trim=True, flags=E.IDENTITY_IDS)
            check_trace(g, trim=True, flags=E.FORCE_REORDER)


def test_c1_gnm_2000_8000():
    g = gen.config("c1")
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    for flags in (0, E.IDENTITY_IDS, E.NO_TRIM, E.SYNC_PASSES, E.NO_DIRTY, E.FORCE_REORDER, E.NO_PACK, E.NO_ASYNC):
        lab, _ = gpu_labels(g, flags)
        np.testing.assert_array_equal(lab, truth)
    check_trace(g, trim=True)
    check_trace(g, trim=False)
    check_trace(g, trim=True, flags=E.IDENTITY_IDS)


# ----------------------------------------------------------------- edge cases
def test_edge_cases():
    # empty graph
    rp = torch.zeros(1, dtype=torch.int32, device="cuda")
    ci = torch.zeros(0, dtype=torch.int32, device="cuda")
    assert E.ecl_scc(rp, ci).numel() == 0
    # no edges
    g = gen.from_edges(7, [])
    np.testing.assert_array_equal(gpu_labels(g)[0], np.arange(7))
    # self-loops and duplicates only
    g = gen.from_edges(5, [(1, 1), (2, 3), (2, 3), (4, 4)])
    np.testing.assert_array_equal(gpu_labels(g)[0], np.arange(5))
    # one directed cycle in random ID order -> one SCC named n-1 (P:247 twist-hex-like)
    n = 100_000
    perm = np.random.default_rng(1).permutation(n)
    g = gen.from_edges(n, np.stack([perm, np.roll(perm, -1)], 1))
    for flags in (0, E.IDENTITY_IDS):
        assert (gpu_labels(g, flags)[0] == n - 1).all()
    # long path (deep DAG): identity
    g = gen.from_edges(n, np.stack([perm[:-1], perm[1:]], 1))
    np.testing.assert_array_equal(gpu_labels(g)[0], np.arange(n))
    # disjoint k-cycles on consecutive IDs
    k = 5
    e = [(b * k + i, b * k + (i + 1) % k) for b in range(1000) for i in range(k)]
    g = gen.from_edges(5000, e)
    v = np.arange(5000)
    np.testing.assert_array_equal(gpu_labels(g)[0], (v // k) * k + k - 1)


def test_heavy_vertices():
    """Hubs far above the warp-cooperation threshold in both directions."""
    rng = np.random.default_rng(5)
    n = 50_000
    hub = 123
    src = np.concatenate([np.full(20_000, hub), rng.integers(0, n, 30_000), rng.integers(0, n, 20_000)])
    dst = np.concatenate([rng.integers(0, n, 20_000), np.full(30_000, 777), rng.integers(0, n, 20_000)])
    g = gen.from_edges(n, np.stack([src, dst], 1))
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    for flags in (0, E.NO_TRIM, E.IDENTITY_IDS):
        np.testing.assert_array_equal(gpu_labels(g, flags)[0], truth)
    check_trace(g, trim=True, max_iters=3)
    # hubs in a graph whose edges all lie inside one 2048-ID range: the pass kernels keep
    # their block-local fixed point (high locality), the long rows go through k_prop_heavy
    n = 2000
    src = np.concatenate([np.full(900, 7), rng.integers(0, n, 900), rng.integers(0, n, 3000)])
    dst = np.concatenate([rng.integers(0, n, 900), np.full(900, 1999), rng.integers(0, n, 3000)])
    g = gen.from_edges(n, np.stack([src, dst], 1))
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    for flags in (0, E.NO_TRIM, E.IDENTITY_IDS):
        np.testing.assert_array_equal(gpu_labels(g, flags)[0], truth)
    check_trace(g, trim=True)


def test_invalid_input_reports_erange():
    rp = torch.tensor([0, 2, 1, 3], dtype=torch.int32, device="cuda")      # decreasing offsets
    ci = torch.tensor([1, 2, 0], dtype=torch.int32, device="cuda")
    with pytest.raises(E.EclSccError) as ex:
        E.ecl_scc(rp, ci)
    assert ex.value.status == E.ERANGE
    rp = torch.tensor([0, 1, 2, 3], dtype=torch.int32, device="cuda")
    ci = torch.tensor([1, 5, 0], dtype=torch.int32, device="cuda")         # column out of range
    with pytest.raises(E.EclSccError) as ex:
        E.ecl_scc(rp, ci)
    assert ex.value.status == E.ERANGE
    plan = E.Plan(2, 2)
    with pytest.raises(E.EclSccError) as ex:                               # plan too small
        E.ecl_scc(rp, torch.tensor([1, 2, 0], dtype=torch.int32, device="cuda"), plan=plan)
    assert ex.value.status == E.EINVAL


def test_host_buffer_entry_point():
    """ecl_scc_host: host CSR in, host labels out (pinned and pageable buffers)."""
    plan = E.Plan(20000, 100000)
    for g in (gen.config("c1"), gen.mesh(12, gen.ordinate(5), kappa=0.2, seed=3), gen.from_edges(9, [])):
        rp, ci = torch.from_numpy(g.row_ptr), torch.from_numpy(g.col_idx)
        truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
        for pin in (False, True):
            a, b = (rp.pin_memory(), ci.pin_memory()) if pin else (rp, ci)
            lab = E.ecl_scc_host(a, b, plan=plan if pin else None)
            np.testing.assert_array_equal(lab.numpy(), truth)


def test_plan_reuse_and_stream():
    g1, g2 = gen.config("c1"), gen.mesh(12, gen.ordinate(7), kappa=0.2, seed=9)
    plan = E.Plan(max(g1.n, g2.n), max(g1.nnz, g2.nnz))
    s = torch.cuda.Stream()
    for g in (g1, g2, g1):
        rp, ci = dev(g)
        torch.cuda.synchronize()
        with torch.cuda.stream(s):
            lab = E.ecl_scc(rp, ci, plan=plan)
        s.synchronize()
        np.testing.assert_array_equal(lab.cpu().numpy(), oracle.tarjan_labels(g.row_ptr, g.col_idx))


# ----------------------------------------------------------------- C2..C5
@pytest.mark.parametrize("order", ["lex", "blocked8"])
def test_c2_mesh_1m(order):
    g = gen.config("c2", order=order)
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    pi = prio(g.n)
    tr = oracle.ecl_scc(*(lambda h: (h.row_ptr, h.col_idx))(relabel(g, pi)), trim=True)
    lab, st = gpu_labels(g)
    np.testing.assert_array_equal(lab, truth)
    assert st["edges_in"] == tr.edges_in[:64] and st["iterations"] == tr.iterations
    assert st["edges_kept"] == tr.edges_kept[:st["iterations"] - 1]
    lab, st = gpu_labels(g, E.IDENTITY_IDS)
    np.testing.assert_array_equal(lab, truth)
    tr = oracle.ecl_scc(g.row_ptr, g.col_idx, trim=True)
    assert st["edges_in"] == tr.edges_in[:64] and st["iterations"] == tr.iterations


def test_c3_rmat_scale22():
    g = gen.config("c3")
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    lab, st = gpu_labels(g)
    np.testing.assert_array_equal(lab, truth)


@pytest.mark.parametrize("order", ["lex", "blocked8"])
def test_c4_mesh_16m(order):
    g = gen.config("c4", order=order)
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    lab, _ = gpu_labels(g)
    np.testing.assert_array_equal(lab, truth)


def test_c5_batched_meshes_full_64():
    """The C5 configuration exactly as bench.py --config c5 times it at N=1: all 64 ordinates
    (131.7M vertices, ~269M edges) in one batched call, every graph's labels compared with
    Tarjan's element by element."""
    from concurrent.futures import ThreadPoolExecutor
    graphs = [gen.config("c5one", order="blocked8", d=d) for d in range(64)]
    dg = [dev(g) for g in graphs]
    plan = E.Plan(sum(g.n for g in graphs), sum(g.nnz for g in graphs), E.NO_VALIDATE)
    labs, st = E.ecl_scc_batched(dg, plan=plan, stats=True)
    torch.cuda.synchronize()
    with ThreadPoolExecutor(max_workers=min(64, os.cpu_count() or 1)) as ex:
        truth = list(ex.map(lambda g: oracle.tarjan_labels(g.row_ptr, g.col_idx), graphs))
    for d, (lab, t) in enumerate(zip(labs, truth)):
        np.testing.assert_array_equal(lab.cpu().numpy(), t, err_msg=f"ordinate {d}")
    # the per-ordinate split of the multi-GPU bench (8 ranks): each share alone, same labels
    for r in (0, 7):
        share = list(range(8 * r, 8 * r + 8))
        sl = E.ecl_scc_batched([dg[d] for d in share])
        torch.cuda.synchronize()
        for d, lab in zip(share, sl):
            np.testing.assert_array_equal(lab.cpu().numpy(), truth[d], err_msg=f"rank {r} ordinate {d}")


def test_batched_host_buffers():
    """ecl_scc_batched_host (the C5 e2e path of bench.py): pinned host CSRs in, host labels
    out, equal to Tarjan's per graph; an empty graph inside the batch; plan reuse."""
    graphs = [gen.mesh(24, gen.ordinate(d), seed=40 + d, order="blocked8", **gen.C4_MESH) for d in range(5)]
    graphs.insert(2, gen.Graph(np.zeros(1, dtype=np.int32), np.zeros(0, dtype=np.int32), "empty"))
    hg = [(torch.from_numpy(g.row_ptr).pin_memory(), torch.from_numpy(g.col_idx).pin_memory()) for g in graphs]
    plan = E.Plan(sum(g.n for g in graphs), sum(g.nnz for g in graphs))
    for _ in range(2):
        labs = E.ecl_scc_batched_host(hg, plan=plan)
        for g, lab in zip(graphs, labs):
            assert lab.device.type == "cpu"
            np.testing.assert_array_equal(lab.numpy(), oracle.tarjan_labels(g.row_ptr, g.col_idx))


def _dense_local_graph(n, seed, back=0.02, span=20):
    """Rows of up to 3 out-edges to the next vertices, one random forward edge and, with
    probability `back`, a short backward edge (small cycles); every row <= 8 entries in both
    directions (so the compaction runs on 4-byte keep words) and almost every vertex with more
    than 4 entries in + out (the overlapped path of k_compact_count2 takes 4, the rest goes
    through trim_mask)."""
    rng = np.random.default_rng(seed)
    indeg = np.zeros(n, dtype=np.int64)
    edges = []
    for v in range(n):
        outs = set()
        for d in (1, 2, 3):
            if rng.random() < 0.85 and v + d < n:
                outs.add(v + d)
        w = v + int(rng.integers(4, 600))
        if w < n:
            outs.add(w)
        if rng.random() < back:
            outs.add(max(0, v - int(rng.integers(1, span))))
        outs.discard(v)
        for w in sorted(outs):
            if indeg[w] < 8:
                edges.append((v, w))
                indeg[w] += 1
    g = gen.from_edges(n, np.array(edges))
    assert np.diff(g.row_ptr).max() <= 8 and indeg.max() <= 8
    return g


@pytest.mark.parametrize("seed", [11, 12])
def test_keep_word_rows_with_more_than_four_entries(seed):
    """Keep-word compaction (rows <= 8) on rows with 5-8 entries: labels and per-iteration
    traces against the oracle (the keep-word count / map kernels, incl. their long-row paths)."""
    g = _dense_local_graph(30000, seed)
    deg = np.diff(g.row_ptr) + np.bincount(g.col_idx, minlength=g.n)
    assert (deg > 4).mean() > 0.5
    lab, _ = gpu_labels(g)
    np.testing.assert_array_equal(lab, oracle.tarjan_labels(g.row_ptr, g.col_idx))
    check_trace(g, trim=True, max_iters=4)


def test_repeated_runs_with_plan_reuse_are_stable():
    """Races show up under repetition: the same plan, several graphs and orders, many runs."""
    graphs = [gen.mesh(60, gen.ordinate(d), seed=4 + d, order=o, **gen.C4_MESH)
              for d, o in ((0, "lex"), (9, "blocked8"), (40, "lex"))]
    plan = E.Plan(max(g.n for g in graphs), max(g.nnz for g in graphs))
    for g in graphs:
        truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
        rp, ci = dev(g)
        for _ in range(4):
            lab = E.ecl_scc(rp, ci, plan=plan)
            torch.cuda.synchronize()
            np.testing.assert_array_equal(lab.cpu().numpy(), truth)


def test_storage_reordering_keeps_labels_and_traces():
    """Graphs without long rows and n >= 16384 are renumbered into BFS-Voronoi cells
    internally (reorder.cuh); labels, per-iteration edge counts and signatures must be
    those of the caller's numbering."""
    g = gen.mesh(16, gen.ordinate(5), seed=7, order="lex", **gen.C4_MESH)    # n = 24576
    truth = oracle.tarjan_labels(g.row_ptr, g.col_idx)
    la, sa = gpu_labels(g, E.FORCE_REORDER)
    lb, sb = gpu_labels(g, E.NO_REORDER)
    np.testing.assert_array_equal(la, truth)
    np.testing.assert_array_equal(lb, truth)
    assert sa["edges_in"] == sb["edges_in"] and sa["iterations"] == sb["iterations"]
    check_trace(g, trim=True, flags=E.FORCE_REORDER, max_iters=3)
    check_trace(g, trim=True, flags=E.IDENTITY_IDS | E.FORCE_REORDER, max_iters=3)
