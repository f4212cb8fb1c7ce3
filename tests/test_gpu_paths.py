"""Every rarely-taken device path is exercised AND bit-exact with the oracle.

The full-size configs run paths that small inputs never reach: hub vertices
processed by a whole CTA, the 64-bit (#nbr, ID) key when #nbr >= 255, the
grid-wide fallback of the cutoff select when a tie group does not fit one
CTA, the forced L = 0 move of the weighted corner case (reading Q8), vertex
deletions in the thread-per-item mode, relocation, compaction.  Each test
below builds an input that forces one of them, runs it through the C ABI
next to the oracle (tests/parity.Pair: partitions, cuts, W_p, stats, delta,
invariants), and asserts with igk_debug_paths that the path really ran.
"""
import numpy as np
import pytest

import igk_inputs as gi
from tests.parity import Pair

pytestmark = pytest.mark.gpu


def _csr_w(n, wedges):
    adj = {u: {} for u in range(n)}
    for u, v, w in wedges:
        adj[u][v] = w
        adj[v][u] = w
    xadj, a, ww = [0], [], []
    for u in range(n):
        for x in sorted(adj[u]):
            a.append(x)
            ww.append(adj[u][x])
        xadj.append(len(a))
    return np.array(xadj, np.int64), np.array(a, np.int32), np.array(ww, np.int32)


def _delta(P, before):
    after = P.G.debug_paths()
    return {k: after[k] - before.get(k, 0) for k in after}


def test_tie_group_grid_fallback_and_cta_select():
    """Isolated vertex insertions all pick the lightest part with #nbr = 0
    (digit 255): one round selects them all, the part overflows, and the
    tie group (every move of that part) has > 4096 members -> grid-wide
    radix passes; a smaller batch fits one CTA."""
    g = gi.make_graph(10_000, 64, 11)
    part = gi.block_partition(g.n, 2)
    P = Pair(g.xadj, g.adjncy, 2, 0.03, part)
    P.refine("settle")
    b0 = P.G.debug_paths()
    assert P.apply(np.array([[2, 0, 0, 1]] * 6000, np.int32), "6000 isolated") == 0
    sto, stg = P.refine("grid tie")
    P.compare_state("grid tie")
    d = _delta(P, b0)
    assert d["tie_grid"] > 0 and d["key_exact"] > 0, d
    b1 = P.G.debug_paths()
    assert P.apply(np.array([[2, 0, 0, 1]] * 1500, np.int32), "1500 isolated") == 0
    P.refine("cta tie")
    P.compare_state("cta tie")
    d = _delta(P, b1)
    assert d["tie_cta"] > 0, d


def test_key64_when_gain_reaches_255():
    """A weighted cycle with edge weight 255 (int = 510 per vertex, so an
    attached new vertex never makes its anchor a candidate); 500 new vertices
    hang on part-0 vertices with weight 255 -> #nbr = 255 (digit 0, the
    non-exact 64-bit key); part 0 overflows -> the cutoff is decided on the
    64-bit keys (grid passes)."""
    n = 4000
    edges = [(i, (i + 1) % n, 255) for i in range(n)]
    xadj, adj, aw = _csr_w(n, edges)
    part = (np.arange(n) >= n // 2).astype(np.int32)
    P = Pair(xadj, adj, 2, 0.03, part, np.ones(n, np.int32), aw)
    P.refine("settle")
    b0 = P.G.debug_paths()
    batch = [[2, 0, 0, 1]] * 500 + [[3, n + j, 1 + j, 255] for j in range(500)]
    assert P.apply(np.array(batch, np.int32), "weighted anchors") == 0
    sto, stg = P.refine("key64")
    P.compare_state("key64", full_csr=True)
    d = _delta(P, b0)
    assert d["key64"] > 0 and stg["moves_deferred"] > 0, (d, stg)


def test_forced_first_move_and_weight_fallback():
    """Weighted corner case (reading Q8): a heavy new vertex fits no part
    (E(u) empty) -> lightest part + imbalance flag; its move alone violates
    the cap -> L = 0 -> forced; IGK_WIMBALANCED on both sides."""
    n = 10
    xadj, adj, aw = _csr_w(n, [(i, i + 1, 1) for i in range(n - 1)])
    part = (np.arange(n) >= 5).astype(np.int32)
    P = Pair(xadj, adj, 2, 0.03, part, np.ones(n, np.int32), aw)
    P.refine("settle")
    b0 = P.G.debug_paths()
    assert P.apply(np.array([[2, 0, 0, 3], [3, 10, 4, 1]], np.int32), "heavy") == 0
    sto, stg = P.refine("forced")
    assert stg["imbalanced"] == 1
    P.compare_state("forced", full_csr=True)
    d = _delta(P, b0)
    assert d["forced_l0"] > 0 and d["wfallback"] > 0, d


def test_restoration_and_clamped_loss_keys():
    """Deleting most of part 1 leaves part 0 far above the shrunken cap:
    R3 evicts with the weighted radix select; a dense part makes the
    restoration threshold fall into a clamped loss digit (int - ext >= 127)."""
    # part 0: a dense block (degree ~ 150, int - ext > 127), part 1: a path
    rng = np.random.default_rng(5)
    n0, n1 = 600, 600
    edges = set()
    for u in range(n0):
        for v in rng.choice(n0, size=75, replace=False):
            if u != v:
                edges.add((min(u, int(v)), max(u, int(v))))
    for u in range(n0, n0 + n1 - 1):
        edges.add((u, u + 1))
    edges.add((0, n0))
    xadj, adj, _ = _csr_w(n0 + n1, [(a, b, 1) for a, b in edges])
    part = np.array([0] * n0 + [1] * n1, np.int32)
    P = Pair(xadj, adj, 2, 0.03, part)
    P.refine("settle")
    b0 = P.G.debug_paths()
    batch = [[1, v, 0, 0] for v in range(n0 + 100, n0 + n1)]
    assert P.apply(np.array(batch, np.int32), "delete part 1") == 0
    sto, stg = P.refine("restore")
    P.compare_state("restore", full_csr=True)
    d = _delta(P, b0)
    assert stg["evicted"] > 0 and d["r3"] > 0 and d["r3_key64"] > 0, (stg, d)


def test_vertex_deletions_thread_mode_and_relocation():
    """> one 8-entry item per warp of the grid: vertex deletions switch to one
    thread per item (the C4 mode); insertions into full prefixes relocate."""
    g = gi.make_graph(60_000, 64, 21)
    part, _ = gi.metis_partition(g, 4)
    P = Pair(g.xadj, g.adjncy, 4, 0.03, part)
    P.refine("settle")
    b0 = P.G.debug_paths()
    S = gi.Stream(g, 8)
    b = S.next(gi.MODE_LITERAL, 0.0, 6000, 100, 100, 3000)
    assert P.apply(b, "many deletions") == 0
    P.refine("many deletions")
    P.compare_state("many deletions", full_csr=True)
    b1 = S.next(gi.MODE_MIX, 0.001)
    assert P.apply(b1, "few deletions") == 0
    P.refine("few deletions")
    P.compare_state("few deletions")
    d = _delta(P, b0)
    assert d["vdel_thread"] > 0 and d["vdel_warp"] > 0 and d["reloc"] > 0, d


def test_hub_paths_counted():
    """A hub (degree > 1024) in A, among the candidates and pending: the CTA
    filter, commit and round gain all run (and match the oracle)."""
    n = 5000
    rng = np.random.default_rng(9)
    edges = {(u, u + 1) for u in range(n - 1)}
    hub = 100
    for v in rng.choice(np.arange(n // 2, n), size=1500, replace=False):
        edges.add((min(hub, int(v)), max(hub, int(v))))
    xadj, adj, _ = _csr_w(n, [(a, b, 1) for a, b in edges])
    part = (np.arange(n) >= n // 2).astype(np.int32)  # the hub sits in part 0, its leaves in part 1
    P = Pair(xadj, adj, 2, 0.5, part)
    b0 = P.G.debug_paths()
    assert P.apply(np.array([[3, hub, 7, 1]], np.int32), "touch hub") == 0
    sto, stg = P.refine("hub")
    P.compare_state("hub", full_csr=True)
    d = _delta(P, b0)
    assert d["hub_filter"] > 0 and d["hub_commit"] > 0 and d["hub_gain"] > 0, (d, stg)


def test_large_insert_batch_compacts_once():
    """Advisor finding (round 1): a batch needing more new slots than a
    default compaction would leave free must still succeed -- the rejected
    validation records the batch's slot demand and the compaction is sized
    by it (one compaction, then the re-run succeeds)."""
    g = gi.make_graph(2000, 16, 31)
    part = gi.block_partition(g.n, 2)
    deg = np.diff(g.xadj)
    used = int((((deg + np.maximum(2, deg // 4)) + 3) & ~3).sum())
    P = Pair(g.xadj, g.adjncy, 2, 0.5, part, max_slots=used + 16)
    P.refine("settle")
    # ~1.4M new directed slots on a 2000-vertex graph (dense insertions among
    # new vertices): far more than the 2 x live + 2^20 a default compaction
    # leaves free on the tiny slab
    nv, win = 2000, 400
    base = g.n
    ii, jj = np.triu_indices(nv, 1)
    keep = (jj - ii) <= win
    ei = np.stack([np.full(keep.sum(), 3), base + ii[keep], base + jj[keep], np.ones(keep.sum())], 1)
    batch = np.concatenate([np.array([[2, 0, 0, 1]] * nv), ei]).astype(np.int32)
    assert 2 * keep.sum() > 2 * used + (1 << 20)
    b0 = P.G.debug_paths()
    assert P.apply(np.array(batch, np.int32), "huge insert") == 0
    P.refine("huge insert")
    P.compare_state("huge insert", full_csr=True)
    d = _delta(P, b0)
    assert d["compaction"] == 1, d


def test_partition_delta_matches_full_vector_changes():
    """igk_partition_delta after igk_step equals the changes of the full
    partition vector (the e2e readback of bench.py)."""
    cfg = gi.CONFIGS["C1"]
    g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(1))
    part, _ = gi.metis_partition(g, 4)
    P = Pair(g.xadj, g.adjncy, 4, cfg["eps"], part, check=False)
    P.refine("settle")
    S = gi.Stream(g, 1234)
    for it in range(5):
        b = S.next(gi.MODE_MIX, 0.03)
        before = P.G.partition()
        assert P.O.apply(b)[0] == 0
        pre = P.O.partition()
        P.O.refine()
        s, st, bad = P.G.step(b)
        assert s == 0
        P.check_delta(pre, f"step {it}")
        after = P.G.partition()
        old = np.full(len(after), -2, np.int32)
        old[: len(before)] = before
        ch = np.nonzero((after >= 0) & (after != old))[0]
        d = P.G.partition_delta()
        assert set(d[:, 0].tolist()) == set(ch.tolist())
        assert np.array_equal(after[d[:, 0]], d[:, 1])
