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


# --------------------------------------------------------------- CPU model of the protocol
def _phase2_partitioned(n, edges, parts, vin, vout):
    """Replicated signatures; each partition relaxes ITS edges to a local fixed point
    (Jacobi), then element-wise MAX over partitions; repeat until no partition changed.
    DESIGN.md reading 12 says the result is the unique global fixed point."""
    exchanges = 0
    while True:
        replicas = []
        changed_any = False
        for es in parts:
            a, b = vin.copy(), vout.copy()
            while True:
                na, nb = a.copy(), b.copy()
                for u, w in es:
                    nb[u] = max(nb[u], b[w])
                    na[w] = max(na[w], a[u])
                if (na == a).all() and (nb == b).all():
                    break
                changed_any = True
                a, b = na, nb
            replicas.append((a, b))
        vin = np.max([r[0] for r in replicas], axis=0)
        vout = np.max([r[1] for r in replicas], axis=0)
        exchanges += 1
        if not changed_any:
            return vin, vout, exchanges


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_partitioned_exchange_reaches_global_fixed_point(P):
    rng = random.Random(10 + P)
    for _ in range(40):
        n = rng.randrange(2, 40)
        edges = [(rng.randrange(n), rng.randrange(n)) for _ in range(rng.randrange(1, 3 * n))]
        edges = [(u, w) for u, w in edges if u != w]
        if not edges:
            continue
        rp, ci = csr_from_edges(n, edges)
        bounds = np.linspace(0, n, P + 1).astype(int)
        parts = [[(u, w) for u, w in edges if bounds[r] <= u < bounds[r + 1]] for r in range(P)]
        vin, vout, _ = _phase2_partitioned(n, edges, parts, np.arange(n), np.arange(n))
        s = oracle.ecl_scc(rp, ci, snap_iter=1)
        np.testing.assert_array_equal(vin, s.snap_in)
        np.testing.assert_array_equal(vout, s.snap_out)
