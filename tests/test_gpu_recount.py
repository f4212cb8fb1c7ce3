"""S9 cut / part-weight reduction on the B200: k_recount3's degree
classes and edge cases against the CPU oracle's cut and W_p, element by
element.  The store is built so that every path of the kernel runs: vertices
counted in-thread (<= 4 entries), through the warp's residual list (5..256),
as one piece (257..1024) and as several pieces (> 1024, a hub of 3000);
a vertex count that is not a multiple of the 128-vertex tile; relocated
prefixes and tombstones (after an applied batch); pending vertices (before
the refine); deleted vertices; unit and weighted handles; the round-1
gather kernel and the TMA variant on the same store (A/B kernels must agree)."""
from __future__ import annotations

import os

import numpy as np
import pytest

import oracle
import paper_conf_dac_leejlczcshh25_b200 as igk

pytestmark = pytest.mark.gpu


def _graph(seed, weighted):
    rng = np.random.default_rng(seed)
    n = 128 * 37 + 5  # ragged last tile
    edges = set()

    def add(u, v):
        if u != v:
            edges.add((min(u, v), max(u, v)))

    for u in range(n):  # a sparse local backbone: degrees 1..6
        for _ in range(rng.integers(0, 3)):
            add(u, (u + int(rng.integers(1, 300))) % n)
    for hub, deg in ((17, 3000), (2222, 700), (4000, 300)):  # several pieces / one piece / one piece
        for v in rng.choice(n, size=deg, replace=False):
            add(hub, int(v))
    for u in range(1000, 1100):  # residual-list vertices (degree ~40)
        for v in rng.choice(n, size=40, replace=False):
            add(u, int(v))
    adj = [[] for _ in range(n)]
    for u, v in sorted(edges):
        adj[u].append(v)
        adj[v].append(u)
    xadj = np.zeros(n + 1, np.int64)
    xadj[1:] = np.cumsum([len(a) for a in adj])
    adjncy = np.array([v for a in adj for v in sorted(a)], np.int32)
    vwgt = adjwgt = None
    if weighted:
        vwgt = rng.integers(1, 5, n).astype(np.int32)
        w = {e: int(rng.integers(1, 9)) for e in edges}
        adjwgt = np.array([w[(min(u, v), max(u, v))] for u in range(n) for v in sorted(adj[u])], np.int32)
    return n, xadj, adjncy, vwgt, adjwgt, rng


def _check(G, O, where):
    cut, wp = G.recount()
    assert cut == O.cut(), (where, cut, O.cut())
    assert np.array_equal(np.asarray(wp), np.asarray(O.part_weights())), where
    return cut


@pytest.mark.parametrize("weighted", [False, True])
def test_recount3_degree_classes_ragged_pending_deleted(weighted):
    n, xadj, adjncy, vwgt, adjwgt, rng = _graph(11 + weighted, weighted)
    assert int(np.diff(xadj).max()) > 1024 and n % 128
    k = 5
    part = rng.integers(0, k, n).astype(np.int32)
    O = oracle.Oracle(xadj, adjncy, k, 0.03, part, vwgt, adjwgt)
    G = igk.IGKGraph(xadj, adjncy, k, 0.03, part, vwgt, adjwgt)
    _check(G, O, "create")
    # a batch that deletes vertices (incl. a neighbour of the big hub),
    # deletes and inserts edges (relocations: the band vertices grow) and
    # inserts vertices (pending until the refine)
    mods = [(1, 5, 0, 0), (1, 300, 0, 0)]
    u = 17
    nb = [int(x) for x in adjncy[xadj[u]:xadj[u + 1]] if int(x) not in (5, 300)]
    mods += [(0, u, nb[3], 0), (0, u, nb[9], 0)]  # (an endpoint deleted in the batch would be invalid)
    have = {(min(a, b), max(a, b)) for a in range(n) for b in adjncy[xadj[a]:xadj[a + 1]]}
    for b in range(1000, 1030):
        for _ in range(12):
            v = int(rng.integers(0, n))
            key = (min(b, v), max(b, v))
            if v != b and v not in (5, 300) and key not in have:
                have.add(key)
                mods.append((3, b, v, int(rng.integers(1, 9)) if weighted else 1))
    mods += [(2, 0, 0, 2 if weighted else 1), (2, 0, 0, 1)]
    mods += [(3, n, 1000, 1), (3, n + 1, 2222, 1)]  # edges of the inserted vertices
    b = np.array(mods, np.int32)
    assert O.apply(b)[0] == 0 and G.apply(b)[0] == 0
    _check(G, O, "after apply (pending + deleted + relocated)")
    O.refine()
    G.refine()
    assert np.array_equal(O.partition(), G.partition())
    _check(G, O, "after refine")


def test_recount_variants_agree():
    """the round-1 gather kernel and the TMA variant (A/B) give k_recount3's result"""
    n, xadj, adjncy, vwgt, adjwgt, rng = _graph(5, False)
    part = rng.integers(0, 4, n).astype(np.int32)
    O = oracle.Oracle(xadj, adjncy, 4, 0.03, part)
    out = {}
    for variant in ("v3", "gather", "tma"):
        os.environ["IGK_RECOUNT"] = variant
        try:
            G = igk.IGKGraph(xadj, adjncy, 4, 0.03, part)
        finally:
            os.environ.pop("IGK_RECOUNT")
        out[variant] = _check(G, O, variant)
        G.close()
    assert len(set(out.values())) == 1


def test_recount_edgeless_and_tiny():
    for n in (1, 3, 129):
        xadj = np.zeros(n + 1, np.int64)
        part = np.arange(n, dtype=np.int32) % 2
        O = oracle.Oracle(xadj, np.zeros(0, np.int32), 2, 0.5, part)
        G = igk.IGKGraph(xadj, np.zeros(0, np.int32), 2, 0.5, part)
        assert _check(G, O, f"edgeless n={n}") == 0
        G.close()
