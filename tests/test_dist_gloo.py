"""Multi-process host logic of the multi-GPU modes on CPU (gloo, world_size 2), and a CPU
model of the partitioned exchange protocol, -m "not gpu"."""
import os
import random
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import gen
import oracle
from oracle import csr_from_edges


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, rp, ci, q):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_alabandisbb23_b200 import dist as D
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    bounds = D.split_rows(world, rp)
    lrp, lci = D.local_csr(rp, ci, bounds[rank], bounds[rank + 1])
    # every rank's rows, gathered, must rebuild the global graph exactly
    parts = [None] * world
    dist.all_gather_object(parts, (bounds[rank], bounds[rank + 1], lrp, lci))
    uid = D.share_unique_id(dist, rank, lambda: os.urandom(128))
    uids = [None] * world
    dist.all_gather_object(uids, uid)
    t = D.max_over_ranks(dist, 1.0 + rank)
    batch = list(D.split_batch(64, world, rank))
    batches = [None] * world
    dist.all_gather_object(batches, batch)
    if rank == 0:
        q.put((bounds, parts, uids, t, batches))
    dist.barrier()
    dist.destroy_process_group()


def test_partition_host_logic_two_ranks_gloo():
    g = gen.mesh(8, gen.ordinate(2), kappa=0.2, seed=3)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, g.row_ptr, g.col_idx, q)) for r in range(2)]
    for p in procs:
        p.start()
    bounds, parts, uids, t, batches = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert bounds[0] == 0 and bounds[-1] == g.n
    rows, cols = [], []
    for rb, re_, lrp, lci in parts:
        assert lrp[0] == 0 and lrp[-1] == len(lci)
        rows.append(np.diff(lrp))
        cols.append(lci)
    np.testing.assert_array_equal(np.concatenate(rows), np.diff(g.row_ptr))
    np.testing.assert_array_equal(np.concatenate(cols), g.col_idx)
    loads = [len(c) for c in cols]
    assert abs(loads[0] - loads[1]) <= 8                       # balanced by edges
    assert uids[0] == uids[1] and len(uids[0]) == 128          # one NCCL id for all ranks
    assert t == 2.0                                            # max over ranks
    assert sorted(batches[0] + batches[1]) == list(range(64))  # batch split covers all graphs


# --------------------------------------------------------------- the halo protocol, on gloo
def halo_protocol(dist, rank, world, rp, ci, trim=True):
    """A plain mirror of run_halo's control flow (driver.cu, halo.cuh) with every exchange a
    real torch.distributed all-reduce (gloo): this rank's rows, its ghosts, the halo H found by
    a MAX all-reduce of ghost marks; per outer iteration Phase 3 on the local edges, the halo's
    kept degrees SUM-reduced for Trim-1, the leave rule (an unfinished, untrimmed halo
    vertex stays), live edges SUM-reduced (termination), and Phase 2 as rounds of local
    Jacobi fixed points whose raised halo copies are MAX-combined until no rank's copy rises;
    finally the owners' labels MAX-reduced.  Signatures are raw IDs (IDENTITY_IDS)."""
    import torch
    from paper_conf_sc_alabandisbb23_b200 import dist as D

    def allreduce(a, op):
        t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.int64))
        dist.all_reduce(t, op=op)
        return t.numpy()

    MAX, SUM = dist.ReduceOp.MAX, dist.ReduceOp.SUM
    n = len(rp) - 1
    bounds = D.split_rows(world, rp)
    rb, re_ = bounds[rank], bounds[rank + 1]
    src = np.repeat(np.arange(rb, re_), np.diff(rp[rb:re_ + 1]))
    dst = np.asarray(ci[rp[rb]:rp[re_]], dtype=np.int64)
    E = np.stack([src, dst], 1)
    E = E[E[:, 0] != E[:, 1]]                               # self-loops add no path
    owned = np.zeros(n, bool)
    owned[rb:re_] = True
    gmark = np.zeros(n, np.int64)
    gmark[E[:, 1][~owned[E[:, 1]]]] = 1
    inH = allreduce(gmark, MAX) > 0
    pos = np.cumsum(inH) - inH
    H = int(inH.sum())
    held = owned | (gmark > 0)
    vin, vout = np.arange(n), np.arange(n)
    alive = held.copy()
    lab = np.full(n, np.iinfo(np.int64).min)
    edges_in = []
    first = True
    while True:
        if not first:                                        # Phase 3
            u, w = E[:, 0], E[:, 1]
            E = E[(vin[u] == vin[w]) & (vout[u] == vout[w]) & (vin[u] != vout[u])]
        kin = np.bincount(E[:, 1], minlength=n)
        kout = np.bincount(E[:, 0], minlength=n)
        trimmed = np.zeros(n, bool)
        if trim:                                             # global degrees of the halo
            hdeg = np.zeros(2 * H, np.int64)
            hv = np.nonzero(held & inH)[0]
            hdeg[2 * pos[hv]], hdeg[2 * pos[hv] + 1] = kin[hv], kout[hv]
            hdeg = allreduce(hdeg, SUM)
            hv = np.nonzero(inH)[0]
            kin[hv], kout[hv] = hdeg[2 * pos[hv]], hdeg[2 * pos[hv] + 1]
            trimmed = (kin == 0) | (kout == 0)
            E = E[~trimmed[E[:, 0]] & ~trimmed[E[:, 1]]]
        deg = np.bincount(E.ravel(), minlength=n) if len(E) else np.zeros(n, np.int64)
        unfinished = np.ones(n, bool) if first else vin != vout
        stay = alive & ((deg > 0) | (inH & unfinished & ~trimmed))
        leave = alive & ~stay
        lab[leave & owned] = np.where(unfinished, np.arange(n), vin)[leave & owned]
        alive = stay
        vin = np.where(alive, np.arange(n), vin)             # Phase 1 for the survivors
        vout = np.where(alive, np.arange(n), vout)
        first = False
        live = int(allreduce(np.array([len(E)]), SUM)[0])
        if live == 0:
            lab[alive & owned] = np.arange(n)[alive & owned]
            break
        edges_in.append(live)
        mine = np.zeros(2 * H, np.int64)                     # this Phase 2's pushes
        while True:
            a0, b0 = vin.copy(), vout.copy()
            while True:                                      # local fixed point (Jacobi)
                na, nb = vin.copy(), vout.copy()
                np.maximum.at(na, E[:, 1], vin[E[:, 0]])
                np.maximum.at(nb, E[:, 0], vout[E[:, 1]])
                if (na == vin).all() and (nb == vout).all():
                    break
                vin, vout = na, nb
            hv = np.nonzero(held & inH & ((vin > a0) | (vout > b0)))[0]
            mine[2 * pos[hv]] = np.maximum(mine[2 * pos[hv]], vin[hv])
            mine[2 * pos[hv] + 1] = np.maximum(mine[2 * pos[hv] + 1], vout[hv])
            hbuf = allreduce(mine, MAX)
            hv = np.nonzero(held & inH)[0]
            xi, xo = hbuf[2 * pos[hv]], hbuf[2 * pos[hv] + 1]
            inj = bool(((xi > vin[hv]) | (xo > vout[hv])).any())
            vin[hv] = np.maximum(vin[hv], xi)
            vout[hv] = np.maximum(vout[hv], xo)
            if not allreduce(np.array([int(inj)]), MAX)[0]:
                break
    return allreduce(lab, MAX), edges_in


def _halo_worker(rank, world, port, graphs, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = [halo_protocol(dist, rank, world, rp, ci, trim=t) for rp, ci, t in graphs]
    if rank == 0:
        q.put(out)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_halo_protocol_gloo(world):
    """The partitioned (halo) protocol with real gloo collectives between `world` processes:
    labels equal Tarjan's, and the live edges per iteration equal O2's (same trim rule) --
    the exchange reaches the global fixed point every iteration (reading 12)."""
    rng = random.Random(31 + world)
    graphs = []
    for k in range(12):
        n = rng.randrange(2, 60)
        edges = [(rng.randrange(n), rng.randrange(n)) for _ in range(rng.randrange(1, 3 * n))]
        rp, ci = csr_from_edges(n, edges)
        graphs.append((rp.astype(np.int32), ci, k % 3 != 0))
    g = gen.mesh(5, gen.ordinate(4), kappa=0.3, seed=2)
    graphs.append((g.row_ptr, g.col_idx, True))
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_halo_worker, args=(r, world, port, graphs, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for (rp, ci, t), (lab, ein) in zip(graphs, res):
        np.testing.assert_array_equal(lab, oracle.tarjan_labels(rp, ci))
        assert ein == oracle.ecl_scc(rp, ci, trim=t).edges_in
