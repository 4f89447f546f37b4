"""Pins for the CPU oracle (oracle/), -m "not gpu".

The oracle is checked against things other than itself (P:n = PAPER.md line n):
  * brute-force reachability (BFS from every vertex, pure Python) on tiny graphs;
  * scipy.sparse.csgraph strong components + max relabel (an independent library);
  * closed forms (P:63 DAG -> all singletons; a single cycle -> one SCC, P:247 twist-hex);
  * invariants of SCCs and of the labels;
  * the hand-derived worked example tests/golden/appendix_a.json;
  * the work bound: at most d outer iterations, d = condensation depth.
"""
import json
import os
import random
from collections import deque

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components

import oracle
from oracle import csr_from_edges

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------- independent helpers
def brute_labels(n, edges):
    """label[v] = max{w : v ~> w and w ~> v}, by BFS from every vertex."""
    adj = [[] for _ in range(n)]
    for u, v in edges:
        adj[u].append(v)
    reach = []
    for s in range(n):
        seen = {s}
        q = deque([s])
        while q:
            x = q.popleft()
            for y in adj[x]:
                if y not in seen:
                    seen.add(y)
                    q.append(y)
        reach.append(seen)
    return np.array([max(w for w in reach[v] if v in reach[w]) for v in range(n)], dtype=np.int32)


def scipy_labels(n, rp, ci):
    a = sp.csr_matrix((np.ones(len(ci), dtype=np.int8), ci, rp), shape=(n, n))
    _, comp = connected_components(a, directed=True, connection="strong")
    mx = np.full(comp.max() + 1 if n else 0, -1, dtype=np.int64)
    np.maximum.at(mx, comp, np.arange(n))
    return mx[comp].astype(np.int32)


def random_edges(rng, n, m, allow_self=True):
    e = []
    for _ in range(m):
        u, v = rng.randrange(n), rng.randrange(n)
        if u == v and not allow_self:
            continue
        e.append((u, v))
    return e


def condensation_depth(n, edges, labels):
    """Longest path (in SCCs) of the condensation, by Kahn's algorithm; None if cyclic."""
    comp = {int(l) for l in labels}
    succ = {c: set() for c in comp}
    indeg = {c: 0 for c in comp}
    for u, v in edges:
        a, b = int(labels[u]), int(labels[v])
        if a != b and b not in succ[a]:
            succ[a].add(b)
            indeg[b] += 1
    level = {c: 1 for c in comp}
    q = deque(c for c in comp if indeg[c] == 0)
    seen = 0
    while q:
        c = q.popleft()
        seen += 1
        for d in succ[c]:
            level[d] = max(level[d], level[c] + 1)
            indeg[d] -= 1
            if indeg[d] == 0:
                q.append(d)
    if seen != len(comp):
        return None
    return max(level.values()) if level else 0


def check_invariants(n, edges, labels):
    labels = np.asarray(labels)
    v = np.arange(n)
    assert (labels >= v).all()                                  # label = max of SCC
    assert (labels[labels] == labels).all()                     # the max names itself
    assert condensation_depth(n, edges, labels) is not None     # condensation is a DAG
    # a vertex of a non-trivial SCC has an in- and an out-neighbour inside it
    size = np.bincount(labels, minlength=n)
    has_in = np.zeros(n, bool)
    has_out = np.zeros(n, bool)
    for a, b in edges:
        if a != b and labels[a] == labels[b]:
            has_out[a] = True
            has_in[b] = True
    nontriv = size[labels] > 1
    assert (has_in[nontriv]).all() and (has_out[nontriv]).all()


FLAGS = [dict(reset_all=r, compress=c, trim=t) for r in (False, True)
         for c in (False, True) for t in (False, True)]


# ---------------------------------------------------------------- O1 Tarjan
def test_tarjan_vs_bruteforce_random():
    rng = random.Random(12345)
    for trial in range(400):
        n = rng.randrange(1, 40)
        m = rng.randrange(0, 3 * n + 1)
        edges = random_edges(rng, n, m)
        rp, ci = csr_from_edges(n, edges)
        got = oracle.tarjan_labels(rp, ci)
        np.testing.assert_array_equal(got, brute_labels(n, edges), err_msg=f"trial {trial}")


def test_tarjan_vs_scipy_larger():
    rng = np.random.default_rng(7)
    for n, m in [(2000, 8000), (20000, 40000), (5000, 5000), (3000, 30000)]:
        u = rng.integers(0, n, m)
        v = rng.integers(0, n, m)
        rp, ci = csr_from_edges(n, np.stack([u, v], 1))
        np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), scipy_labels(n, rp, ci))


def test_tarjan_deep_path_no_recursion_limit():
    # a 200k-long cycle exercises the explicit frame stack (recursive DFS would overflow)
    n = 200_000
    perm = np.random.default_rng(3).permutation(n)
    edges = np.stack([perm, np.roll(perm, -1)], 1)
    rp, ci = csr_from_edges(n, edges)
    assert (oracle.tarjan_labels(rp, ci) == n - 1).all()
    # and a path in random order: all singletons
    rp, ci = csr_from_edges(n, edges[:-1])
    np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), np.arange(n))


def test_closed_forms():
    rng = np.random.default_rng(11)
    for n in (1, 2, 17, 1000):
        perm = rng.permutation(n)
        # DAG with random IDs: every SCC trivial -> identity
        a = rng.integers(0, n, 4 * n)
        b = rng.integers(0, n, 4 * n)
        lo, hi = np.minimum(a, b), np.maximum(a, b)
        keep = lo < hi
        dag = np.stack([perm[lo[keep]], perm[hi[keep]]], 1)
        rp, ci = csr_from_edges(n, dag)
        np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), np.arange(n))
        # complete digraph: one SCC named n-1
        if n <= 200:
            e = [(i, j) for i in range(n) for j in range(n) if i != j]
            rp, ci = csr_from_edges(n, e)
            assert (oracle.tarjan_labels(rp, ci) == n - 1).all()
    # disjoint k-cycles on consecutive IDs: label = floor(v/k)*k + k-1
    for k in (2, 3, 7):
        n = 10 * k
        e = [(g * k + i, g * k + (i + 1) % k) for g in range(10) for i in range(k)]
        rp, ci = csr_from_edges(n, e)
        v = np.arange(n)
        np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), (v // k) * k + k - 1)


def test_empty_and_isolated():
    rp, ci = csr_from_edges(5, [])
    np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), np.arange(5))
    tr = oracle.ecl_scc(rp, ci)
    np.testing.assert_array_equal(tr.labels, np.arange(5))
    assert tr.iterations == 0
    rp, ci = csr_from_edges(3, [(1, 1), (1, 1)])       # self-loops and duplicates only
    np.testing.assert_array_equal(oracle.ecl_scc(rp, ci).labels, np.arange(3))
    np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), np.arange(3))


def test_invariants_random():
    rng = random.Random(99)
    for _ in range(100):
        n = rng.randrange(1, 60)
        edges = random_edges(rng, n, rng.randrange(0, 3 * n))
        rp, ci = csr_from_edges(n, edges)
        check_invariants(n, edges, oracle.tarjan_labels(rp, ci))


# ---------------------------------------------------------------- O2 plain ECL-SCC
def test_appendix_a_labels_and_traces():
    g = json.load(open(os.path.join(GOLDEN, "appendix_a.json")))
    n, edges = g["n"], g["edges"]
    rp, ci = csr_from_edges(n, edges)
    np.testing.assert_array_equal(brute_labels(n, edges), g["labels"])
    np.testing.assert_array_equal(oracle.tarjan_labels(rp, ci), g["labels"])
    for key, trim in (("r2_no_trim", False), ("r2_trim1", True)):
        exp = g[key]
        for compress in (False, True):
            tr = oracle.ecl_scc(rp, ci, trim=trim, compress=compress)
            np.testing.assert_array_equal(tr.labels, g["labels"])
            assert tr.edges_in == exp["edges_in"], (key, compress)
            assert tr.edges_kept == exp["edges_kept"], (key, compress)
            if not compress:
                assert tr.passes == exp["passes_jacobi"], key
            for it in range(1, tr.iterations + 1):
                s = oracle.ecl_scc(rp, ci, trim=trim, compress=compress, snap_iter=it)
                np.testing.assert_array_equal(s.snap_in, exp["in"][it - 1], err_msg=f"{key} it{it}")
                np.testing.assert_array_equal(s.snap_out, exp["out"][it - 1], err_msg=f"{key} it{it}")
    # iteration 1 splits the left "linked list" cluster into 4 pieces
    s = oracle.ecl_scc(rp, ci, snap_iter=1)
    left = [0, 1, 2, 3, 4, 6, 9]
    assert len({(s.snap_in[v], s.snap_out[v]) for v in left}) == 4
    # max SCCs of the two clusters (containing 9 and 11) finish in iteration 1
    for v in (4, 9, 11):
        assert s.snap_in[v] == s.snap_out[v]


@pytest.mark.parametrize("flags", FLAGS, ids=lambda f: "-".join(k for k, v in f.items() if v) or "r2")
def test_ecl_scc_matches_tarjan_random(flags):
    rng = random.Random(2024)
    for trial in range(300):
        n = rng.randrange(1, 40)
        edges = random_edges(rng, n, rng.randrange(0, 3 * n + 1))
        rp, ci = csr_from_edges(n, edges)
        tr = oracle.ecl_scc(rp, ci, **flags)
        np.testing.assert_array_equal(tr.labels, oracle.tarjan_labels(rp, ci),
                                      err_msg=f"trial {trial} {flags}")


def test_ecl_scc_matches_tarjan_larger():
    rng = np.random.default_rng(5)
    for n, m in [(2000, 8000), (3000, 3300), (1500, 9000)]:
        rp, ci = csr_from_edges(n, np.stack([rng.integers(0, n, m), rng.integers(0, n, m)], 1))
        truth = scipy_labels(n, rp, ci)
        for trim in (False, True):
            np.testing.assert_array_equal(oracle.ecl_scc(rp, ci, trim=trim, compress=True).labels, truth)


def test_iteration_bound_dag_depth():
    """the outer loop runs at most d times, d = depth of the condensation DAG."""
    rng = random.Random(7)
    for _ in range(300):
        n = rng.randrange(1, 30)
        edges = random_edges(rng, n, rng.randrange(0, 2 * n + 1))
        rp, ci = csr_from_edges(n, edges)
        truth = oracle.tarjan_labels(rp, ci)
        d = condensation_depth(n, edges, truth)
        for trim in (False, True):
            assert oracle.ecl_scc(rp, ci, trim=trim).iterations <= d


def test_trace_independent_of_compression():
    """DESIGN.md reading 12: Phase 2's fixed point is unique, so path compression changes
    pass counts only -- never edges_in/edges_kept or the signatures after Phase 2."""
    rng = random.Random(31)
    for _ in range(100):
        n = rng.randrange(2, 40)
        edges = random_edges(rng, n, rng.randrange(0, 3 * n))
        rp, ci = csr_from_edges(n, edges)
        for trim in (False, True):
            a = oracle.ecl_scc(rp, ci, trim=trim)
            b = oracle.ecl_scc(rp, ci, trim=trim, compress=True)
            assert a.edges_in == b.edges_in and a.edges_kept == b.edges_kept
            for it in range(1, a.iterations + 1):
                sa = oracle.ecl_scc(rp, ci, trim=trim, snap_iter=it)
                sb = oracle.ecl_scc(rp, ci, trim=trim, compress=True, snap_iter=it)
                np.testing.assert_array_equal(sa.snap_in, sb.snap_in)
                np.testing.assert_array_equal(sa.snap_out, sb.snap_out)


def test_phase2_fixed_point_is_reachability_max():
    """After Phase 2 of iteration 1: in[v] = max ancestor (incl. v), out[v] = max
    descendant, checked by BFS."""
    rng = random.Random(4)
    for _ in range(100):
        n = rng.randrange(1, 40)
        edges = random_edges(rng, n, rng.randrange(0, 3 * n))
        rp, ci = csr_from_edges(n, edges)
        s = oracle.ecl_scc(rp, ci, snap_iter=1)
        if s.iterations == 0:
            continue
        fwd = [[] for _ in range(n)]
        for u, v in edges:
            fwd[u].append(v)
        reach = []
        for v in range(n):
            seen, q = {v}, deque([v])
            while q:
                x = q.popleft()
                for y in fwd[x]:
                    if y not in seen:
                        seen.add(y)
                        q.append(y)
            reach.append(seen)
        for v in range(n):
            assert s.snap_out[v] == max(reach[v])
            assert s.snap_in[v] == max(w for w in range(n) if v in reach[w])


# ---------------------------------------------------------------- Appendix B readings
def _literal_p190(n, edges):
    """The literal reading of P:190 ('before overwriting signature s of v with a larger t,
    also update vertex s's signature with t'), on top of R2 + Jacobi-free sequential
    relaxation.  Written here only to show it is unsound (reading 5)."""
    vin = list(range(n)); vout = list(range(n))
    E = [(u, v) for u, v in edges if u != v]
    while E:
        changed = True
        while changed:
            changed = False
            for u, v in E:
                if vout[v] > vout[u]:
                    s, t = vout[u], vout[v]
                    if t > vout[s]:
                        vout[s] = t
                    vout[u] = t; changed = True
                if vin[u] > vin[v]:
                    s, t = vin[v], vin[u]
                    if t > vin[s]:
                        vin[s] = t
                    vin[v] = t; changed = True
        E = [(u, v) for u, v in E if vin[u] == vin[v] and vout[u] == vout[v] and vin[u] != vout[u]]
        for x in range(n):
            if vin[x] != vout[x]:
                vin[x] = vout[x] = x
    return vin


def test_p190_literal_reading_is_unsound_and_excluded():
    n, edges = 10, [(5, 2), (5, 9), (9, 2)]
    rp, ci = csr_from_edges(n, edges)
    truth = oracle.tarjan_labels(rp, ci)
    assert truth[5] == 5
    assert _literal_p190(n, edges)[5] == 9          # literal trick gives a wrong label
    assert oracle.ecl_scc(rp, ci).labels[5] == 5     # the oracle does not implement it


def test_p169_claim_counterexample():
    """P:169 says all non-max SCCs have in != out after Phase 2; with edges {5->3, 9->3}
    vertex 5 reaches (5,5) in iteration 1 although its cluster's max SCC is {9}."""
    rp, ci = csr_from_edges(10, [(5, 3), (9, 3)])
    s = oracle.ecl_scc(rp, ci, snap_iter=1)
    assert s.snap_in[5] == 5 and s.snap_out[5] == 5
    np.testing.assert_array_equal(s.labels, np.arange(10))


# ---------------------------------------------------------------- O4: sweep levels
def brute_levels(n, edges, labels):
    """level of each vertex's SCC = longest condensation path ending there, by enumerating
    every path from every SCC with a depth-first search (exponential: tiny graphs only)."""
    comps = sorted({int(l) for l in labels})
    succ = {c: set() for c in comps}
    for u, v in edges:
        a, b = int(labels[u]), int(labels[v])
        if a != b:
            succ[a].add(b)
    best = {c: 0 for c in comps}

    def walk(c, length):
        best[c] = max(best[c], length)
        for d in succ[c]:
            walk(d, length + 1)

    for c in comps:
        walk(c, 0)
    return np.array([best[int(labels[v])] for v in range(n)], dtype=np.int32)


def test_levels_vs_bruteforce_paths():
    rng = random.Random(11)
    for trial in range(300):
        n = rng.randrange(1, 11)
        edges = random_edges(rng, n, rng.randrange(0, 2 * n + 1))
        rp, ci = csr_from_edges(n, edges)
        lab = brute_labels(n, edges)
        lv, depth = oracle.scc_levels(rp, ci, lab)
        exp = brute_levels(n, edges, lab)
        np.testing.assert_array_equal(lv, exp, err_msg=f"trial {trial}")
        assert depth == exp.max() + 1


def test_levels_closed_forms_and_invariants():
    rng = np.random.default_rng(3)
    # a path in random ID order: level = position on the path
    n = 5000
    perm = rng.permutation(n)
    rp, ci = csr_from_edges(n, np.stack([perm[:-1], perm[1:]], 1))
    lv, depth = oracle.scc_levels(rp, ci, np.arange(n))
    pos = np.empty(n, dtype=np.int32)
    pos[perm] = np.arange(n)
    np.testing.assert_array_equal(lv, pos)
    assert depth == n
    # disjoint cycles: every SCC is a source
    k = 7
    e = [(b * k + i, b * k + (i + 1) % k) for b in range(50) for i in range(k)]
    rp, ci = csr_from_edges(350, e)
    lv, depth = oracle.scc_levels(rp, ci, oracle.tarjan_labels(rp, ci))
    assert (lv == 0).all() and depth == 1
    # a chain of 3-cycles: cycle j has level j
    e = [(3 * j + i, 3 * j + (i + 1) % 3) for j in range(40) for i in range(3)] + \
        [(3 * j + 2, 3 * (j + 1)) for j in range(39)]
    rp, ci = csr_from_edges(120, e)
    lv, depth = oracle.scc_levels(rp, ci, oracle.tarjan_labels(rp, ci))
    np.testing.assert_array_equal(lv, np.arange(120) // 3)
    assert depth == 40
    # invariants on random graphs: every inter-SCC edge climbs >= 1 level; every SCC above
    # level 0 has a predecessor exactly one level below (the longest path is tight)
    r = random.Random(5)
    for _ in range(20):
        n = r.randrange(50, 400)
        edges = random_edges(r, n, r.randrange(0, 3 * n))
        rp, ci = csr_from_edges(n, edges)
        lab = oracle.tarjan_labels(rp, ci)
        lv, depth = oracle.scc_levels(rp, ci, lab)
        tight = np.zeros(n, bool)
        for u, v in edges:
            if lab[u] != lab[v]:
                assert lv[v] >= lv[u] + 1
                if lv[v] == lv[u] + 1:
                    tight[lab[v]] = True
        reps = np.unique(lab)
        assert all(tight[c] for c in reps if lv[c] > 0)
        assert depth == lv.max() + 1 == condensation_depth(n, edges, lab)


def test_levels_reject_cyclic_labels():
    rp, ci = csr_from_edges(3, [(0, 1), (1, 0)])
    with pytest.raises(ValueError):
        oracle.scc_levels(rp, ci, np.array([0, 1, 2]))       # 0 and 1 labelled apart: a cycle


# ---------------------------------------------------------------- variants (f2, f3)
def _brute_variant(n, edges, trim=False, trim2=False, four=False):
    """Rule R2 iterated by DEFINITION, not by propagation: after the trims, every live
    vertex's signatures are the max (and, with four, min) vertex ID over its ancestors and
    over its descendants in the live edge set, by BFS; Phase 3
    keeps an edge iff all signatures agree at both ends and its source is unfinished
    (P:147).  Trim-1 drops the edges of a vertex without live in- or out-edges;
    Trim-2 finishes a pair u<->w whose only live in-edge entries (or only out-edge entries)
    come from each other.  Returns (labels, edges_in, edges_kept)."""
    E = [(u, v) for u, v in edges if u != v]
    label = list(range(n))
    edges_in, kept = [], []
    while True:
        if trim or trim2:
            din, dout = [0] * n, [0] * n
            ins, outs = [[] for _ in range(n)], [[] for _ in range(n)]
            for u, v in E:
                dout[u] += 1; din[v] += 1
                outs[u].append(v); ins[v].append(u)
            pair = [-1] * n
            if trim2:
                for u in range(n):
                    if din[u] == 1 and din[ins[u][0]] == 1 and ins[ins[u][0]][0] == u:
                        pair[u] = ins[u][0]
                    if dout[u] == 1 and dout[outs[u][0]] == 1 and outs[outs[u][0]][0] == u:
                        pair[u] = outs[u][0]
            gone = [(trim and (din[x] == 0 or dout[x] == 0)) or pair[x] >= 0 for x in range(n)]
            E = [(u, v) for u, v in E if not gone[u] and not gone[v]]
            for u in range(n):
                if pair[u] >= 0:
                    label[u] = max(u, pair[u])
        if not E:
            break
        edges_in.append(len(E))
        fwd = [[] for _ in range(n)]
        for u, v in E:
            fwd[u].append(v)
        reach = []
        for s in range(n):
            seen, q = {s}, deque([s])
            while q:
                x = q.popleft()
                for y in fwd[x]:
                    if y not in seen:
                        seen.add(y)
                        q.append(y)
            reach.append(seen)
        anc = [[w for w in range(n) if v in reach[w]] for v in range(n)]
        sig = [(max(anc[v]), max(reach[v])) + ((min(anc[v]), min(reach[v])) if four else ()) for v in range(n)]
        E = [(u, v) for u, v in E if sig[u] == sig[v] and sig[u][0] != sig[u][1]]
        kept.append(len(E))
        live = {x for e in E for x in e}
        for v in range(n):
            if sig[v][0] == sig[v][1] and (v in live or any(v in e for e in edges)):
                label[v] = sig[v][0] if label[v] == v else label[v]
    return np.array(label, dtype=np.int32), edges_in, kept


VARIANTS = [dict(trim2=True), dict(trim=True, trim2=True), dict(four=True), dict(four=True, trim=True),
            dict(four=True, trim=True, trim2=True), dict(raise_=True), dict(raise_=True, trim=True),
            dict(raise_=True, compress=True, trim=True, trim2=True, four=True)]


@pytest.mark.parametrize("flags", VARIANTS, ids=lambda f: "-".join(k for k in f))
def test_variants_labels_and_traces_vs_brute_force(flags):
    """O2 with Trim-2 / 4 signatures / the sound P:190 trick against the brute-force
    definition above (labels, live edges per iteration, kept edges), and against Tarjan."""
    rng = random.Random(606)
    bf = {k: v for k, v in flags.items() if k in ("trim", "trim2", "four")}
    for trial in range(250):
        n = rng.randrange(1, 30)
        edges = random_edges(rng, n, rng.randrange(0, 3 * n + 1))
        if trial % 3 == 0:                       # plant 2-cycles (Trim-2 candidates)
            for _ in range(3):
                a, b = rng.randrange(n), rng.randrange(n)
                edges += [(a, b), (b, a)]
        rp, ci = csr_from_edges(n, edges)
        tr = oracle.ecl_scc(rp, ci, **flags)
        truth = oracle.tarjan_labels(rp, ci)
        np.testing.assert_array_equal(tr.labels, truth, err_msg=f"trial {trial}")
        lab, ein, kept = _brute_variant(n, edges, **bf)
        np.testing.assert_array_equal(lab, truth, err_msg=f"brute trial {trial}")
        assert tr.edges_in == ein and tr.edges_kept == kept, (trial, tr.edges_in, ein, tr.edges_kept, kept)


def test_trim2_hand_examples():
    """'Any two vertices that have no incoming or outgoing edges aside from a
    bidirectional edge connecting them to each other' form an SCC."""
    # {0<->1} whose only out-edges are each other, fed by 2: Trim-1 takes 2, Trim-2 {0,1};
    # no live edge is left, so Phase 2 never runs (0 iterations)
    rp, ci = csr_from_edges(3, [(0, 1), (1, 0), (2, 0)])
    for trim in (False, True):
        tr = oracle.ecl_scc(rp, ci, trim=trim, trim2=True)
        assert tr.labels.tolist() == [1, 1, 2] and tr.iterations == 0
    # the same pair with one extra in-edge AND one extra out-edge: no pattern applies
    rp, ci = csr_from_edges(5, [(0, 1), (1, 0), (2, 0), (1, 4), (4, 2)])
    tr = oracle.ecl_scc(rp, ci, trim2=True)
    assert tr.iterations >= 1 and tr.labels.tolist() == [4, 4, 4, 3, 4]
    # duplicate edges are counted: 0->1 twice gives 1 two in-edge entries (reading 17)
    rp, ci = csr_from_edges(2, [(0, 1), (0, 1), (1, 0)])
    tr = oracle.ecl_scc(rp, ci, trim2=True)
    assert tr.labels.tolist() == [1, 1]
    assert tr.edges_in[0] == 3                        # out-pattern: dout[0] = 2, in: din[1] = 2
    with pytest.raises(ValueError):
        oracle.ecl_scc(rp, ci, trim2=True, reset_all=True)


def test_four_signatures_hand_example():
    """the minimums separate SCCs the maximums cannot.  Path 5 -> 0 -> 9 (no trim):
    with two signatures 5 and 0 share (in, out) = (5, 9) and their edge survives iteration 1;
    the minimums give 5: (min in, min out) = (5, 0) and 0: (0, 0), so it is removed."""
    rp, ci = csr_from_edges(10, [(5, 0), (0, 9)])
    base = oracle.ecl_scc(rp, ci)
    assert base.edges_in == [2, 1] and base.edges_kept == [1, 0]
    four = oracle.ecl_scc(rp, ci, four=True)
    assert four.edges_in == [2] and four.edges_kept == [0]
    np.testing.assert_array_equal(four.labels, np.arange(10))


def test_sound_p190_variant_keeps_the_trace_and_cuts_passes():
    """The sound P:190 variant changes pass counts only (reading 12): same signatures after
    every Phase 2; on a long cycle in random ID order it needs fewer Jacobi rounds; the
    Appendix B counterexample to the literal reading stays correct."""
    rng = random.Random(12)
    for _ in range(60):
        n = rng.randrange(2, 40)
        edges = random_edges(rng, n, rng.randrange(0, 3 * n))
        rp, ci = csr_from_edges(n, edges)
        a = oracle.ecl_scc(rp, ci, trim=True)
        b = oracle.ecl_scc(rp, ci, trim=True, raise_=True)
        assert a.edges_in == b.edges_in and a.edges_kept == b.edges_kept
        for it in range(1, a.iterations + 1):
            sa = oracle.ecl_scc(rp, ci, trim=True, snap_iter=it)
            sb = oracle.ecl_scc(rp, ci, trim=True, raise_=True, snap_iter=it)
            np.testing.assert_array_equal(sa.snap_in, sb.snap_in)
            np.testing.assert_array_equal(sa.snap_out, sb.snap_out)
    perm = np.random.default_rng(3).permutation(4096)
    rp, ci = csr_from_edges(4096, np.stack([perm, np.roll(perm, -1)], 1))
    assert oracle.ecl_scc(rp, ci, raise_=True).passes[0] < oracle.ecl_scc(rp, ci).passes[0]
    rp, ci = csr_from_edges(10, [(5, 2), (5, 9), (9, 2)])
    assert oracle.ecl_scc(rp, ci, raise_=True).labels[5] == 5
