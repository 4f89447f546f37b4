"""Host model of the asynchronous Phase-2 tile queue (pack.cuh AsyncQ: aq_mark, the claim,
aq_finish) under random interleavings of atomic steps.

The kernel's termination test is `pending == 0`.  With the round-2 accounting, pending counts
dirty tiles once, running tiles once and running-and-dirtied-again tiles twice, so a mark that
changes a state adds one and every finish subtracts one (two fire-and-forget reductions).  The
model replays the same per-thread atomic step sequences the device code issues -- the finish
as two separately scheduled reductions, a mark as compare-and-swap attempts followed by a
separate increment -- and checks that pending is exact whenever no visit is in flight, that a
visit's own marks are counted before its finish lands (so the marking CTA, which reads pending
after its fence, never exits while a tile it dirtied is unclaimed), and that draining always
ends with every tile clean.  (As in round 1, another CTA may read a transient zero while a
mark's increment is in flight and leave early; the marking CTA finishes that work.)  Runs on
CPU (no GPU)."""
import random

import pytest


class Queue:
    def __init__(self, ntiles):
        self.state = [1] * ntiles          # k_async_init: every tile dirty
        self.pending = ntiles

    def work_left(self):
        # tiles still to be visited (dirty) or being visited; a running-and-dirtied tile needs its
        # current visit and one more
        return sum({0: 0, 1: 1, 2: 1, 3: 2}[s] for s in self.state)


def mark_steps(q, t):
    """aq_mark as a generator of atomic steps: CAS 0->1 first, else 2->3, then pending += 1."""
    st = 0
    while True:
        old = q.state[t]
        if old == st:
            q.state[t] = 1 if st == 0 else 3
            yield
            break
        yield
        if old in (1, 3):
            return
        st = old
    q.pending += 1
    yield


def finish_steps(q, t, v):
    """aq_finish: state -= 2 and pending -= 1 as two independent reductions (either order)."""
    first = random.random() < 0.5
    for k in range(2):
        if (k == 0) == first:
            q.state[t] -= 2
        else:
            q.pending -= 1
            v["dec"] = True
        yield


def visit_steps(q, t, marks, v):
    # the visit's marks all complete (fence + barrier) before its finish is issued
    for m in marks:
        yield from mark_steps(q, m)
    v["marked"] = marks
    yield from finish_steps(q, t, v)


@pytest.mark.parametrize("seed", range(40))
def test_pending_never_undercounts_and_is_exact_at_quiescence(seed):
    random.seed(seed)
    nt = random.randint(2, 9)
    q = Queue(nt)
    running = []                                   # generators of in-flight visits
    for _ in range(4000):
        # a claimer takes a dirty tile (1 -> 2) when one exists
        if random.random() < 0.35:
            dirty = [t for t in range(nt) if q.state[t] == 1]
            if dirty and len(running) < 4:
                t = random.choice(dirty)
                q.state[t] = 2
                # a visit marks the tiles of its cut edges: never its own tile
                others = [u for u in range(nt) if u != t]
                marks = random.sample(others, random.randint(0, min(3, len(others)))) if random.random() < 0.6 else []
                v = {"dec": False}
                running.append((visit_steps(q, t, marks, v), v))
        if running:
            g = random.choice(running)
            try:
                next(g[0])
            except StopIteration:
                running.remove(g)
        # the marking visit, once all its marks are counted (its fence), sees pending >= the
        # tiles it dirtied that are still dirty
        for _, v in running:
            if v.get("marked") is not None and not v["dec"]:
                assert q.pending >= sum(1 for u in v["marked"] if q.state[u] in (1, 3)), (q.state, q.pending)
        if not running:
            assert q.pending == q.work_left(), (q.state, q.pending)
    # drain: finish every visit, then every dirty tile with visits that mark nothing
    while running:
        g = running[0]
        try:
            next(g[0])
        except StopIteration:
            running.pop(0)
    while q.pending:
        t = next(t for t in range(nt) if q.state[t] == 1)
        q.state[t] = 2
        for _ in visit_steps(q, t, [], {"dec": False}):
            pass
    assert all(s == 0 for s in q.state)
