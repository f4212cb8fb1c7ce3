"""NEXT-2 parity: the GPU full partitioner igk_fgp_partition (IGK-FGP v1,
csrc/fgp.cuh + igk.cu) vs the oracle's ora_fgp (oracle/igk_fgp.c), bit-exact
on the partition vector and the level sizes.

Graphs: random (unit / weighted / tie-heavy), grids, the circuit generator
(unit and weighted, 20K and 200K vertices), isolated vertices, graphs below
35 k vertices (no coarsening), group sizes 2 / 3 / 6, k in {2, 3, 4, 8, 16, 64}.
"""
import numpy as np
import pytest

import igk_inputs as gi
import oracle
import paper_conf_dac_leejlczcshh25_b200 as igk
from tests.test_oracle_fgp import csr_from_edges, cut_of, grid_graph, random_graph


def _both(xadj, adj, k, eps=0.03, vwgt=None, adjwgt=None, s=6):
    po, lo = oracle.fgp(xadj, adj, k, eps, vwgt=vwgt, adjwgt=adjwgt, group_size=s)
    pg, lg = igk.fgp_partition(xadj, adj, k, eps, vwgt=vwgt, adjwgt=adjwgt, group_size=s)
    assert lg == lo, (lg, lo)
    mism = np.flatnonzero(po != pg)
    assert mism.size == 0, f"{mism.size} vertices differ, first {mism[:8]}"
    return pg, lg


@pytest.mark.gpu
@pytest.mark.parametrize("s", [2, 3, 6])
@pytest.mark.parametrize("name,k", [("rand_unit", 2), ("rand_w", 4), ("rand_ties", 3), ("grid", 4)])
def test_small_graphs(name, k, s):
    if name == "grid":
        xadj, adj, _ = grid_graph(40, 50)
        aw = None
    else:
        n, m, seed, wmax = {"rand_unit": (3000, 7000, 1, 1), "rand_w": (4000, 10000, 2, 9),
                            "rand_ties": (5000, 6000, 3, 2)}[name]
        xadj, adj, aw = random_graph(n, m, seed, wmax)
        if wmax == 1:
            aw = None
    _both(xadj, adj, k, adjwgt=aw, s=s)


@pytest.mark.gpu
@pytest.mark.parametrize("k", [2, 4, 16, 64])
def test_circuit_20k(k):
    g = gi.make_graph(20000, 64, 3)
    part, lv = _both(g.xadj, g.adjncy, k)
    assert len(lv) >= 2


@pytest.mark.gpu
def test_circuit_weighted():
    g = gi.make_graph(30000, 256, 7, weighted=True)
    _both(g.xadj, g.adjncy, 8, vwgt=g.vwgt, adjwgt=g.adjwgt)


@pytest.mark.gpu
def test_circuit_200k():
    g = gi.make_graph(200000, 1024, 21)
    part, lv = _both(g.xadj, g.adjncy, 8)
    assert lv[0] == 200000 and len(lv) >= 4


@pytest.mark.gpu
@pytest.mark.parametrize("k", [2, 8])
def test_no_coarsening_and_isolated(k):
    # below 35 k vertices: one level
    xadj, adj, aw = random_graph(30 * k, 50 * k, 5)
    _, lv = _both(xadj, adj, k, adjwgt=aw)
    assert lv == [30 * k]
    # many isolated vertices: < 90% coarsenable after one level at most
    edges = {(2 * i, 2 * i + 1): 1 for i in range(300)}
    xadj, adj, aw = csr_from_edges(2000, edges)
    _both(xadj, adj, k, adjwgt=aw)
    # no edges at all
    xadj = np.zeros(501, np.int64)
    _both(xadj, np.zeros(0, np.int32), k)


@pytest.mark.gpu
def test_eps_and_balance():
    g = gi.make_graph(50000, 64, 8)
    for eps in (0.01, 0.1):
        part, _ = _both(g.xadj, g.adjncy, 4, eps=eps)
        pw = np.bincount(part, minlength=4)
        assert pw.max() <= oracle.cap(g.n, eps, 4)


@pytest.mark.gpu
def test_invalid():
    xadj, adj, aw = random_graph(100, 200, 1)
    for kw in ({"k": 1}, {"k": 2, "group_size": 1}, {"k": 2, "eps": 0.0}):
        k = kw.pop("k")
        with pytest.raises(igk.IGKError):
            igk.fgp_partition(xadj, adj, k, kw.pop("eps", 0.03), **kw)
    bad = adj.copy()
    bad[0] = 0 if bad[0] != 0 else 1  # breaks symmetry / adds a self loop
    with pytest.raises(igk.IGKError):
        igk.fgp_partition(xadj, bad, 2, 0.03)


def test_invalid_host_side():
    """rejected before any device work (runs without a GPU)"""
    xadj, adj, aw = random_graph(100, 200, 1)
    for k, s, eps in ((1, 6, 0.03), (2, 1, 0.03), (2, 6, 0.0), (2, 6, 2.0)):
        with pytest.raises(igk.IGKError):
            igk.fgp_partition(xadj, adj, k, eps, group_size=s)


# ---- F8 / F9: repartition of a live handle, fallback policy -----------------------
from tests.parity import Pair  # noqa: E402


def _c1_pair(k=4, **kw):
    cfg = gi.CONFIGS["C1"]
    g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(0))
    part, _ = gi.metis_partition(g, k)
    P = Pair(g.xadj, g.adjncy, k, cfg["eps"], part, **kw)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(0)))
    return cfg, P, S


@pytest.mark.gpu
def test_repartition_parity_mid_stream():
    cfg, P, S = _c1_pair()
    for it in range(cfg["iters"]):
        assert P.apply(gi.next_batch(S, cfg), f"it{it}") == 0
        P.refine(f"it{it}")
        if it in (4, 12):
            P.repartition(f"repartition after it{it}")
            with pytest.raises(igk.IGKError):
                P.G.partition_delta()
    P.compare_state("end", full_csr=True)


@pytest.mark.gpu
def test_repartition_refuses_pending():
    cfg, P, S = _c1_pair()
    assert P.apply(gi.next_batch(S, cfg)) == 0
    with pytest.raises(igk.IGKError) as e:
        P.G.repartition()
    assert e.value.status == 5
    P.refine()
    P.repartition()


@pytest.mark.gpu
def test_fallback_policy():
    """fgp_fallback = 15%: the handle repartitions by itself once the accepted
    modifiers (600 per C1 batch) reach 15% of |V| at the last full partition;
    the oracle side applies the same rule here (reading F9)"""
    cfg, P, S = _c1_pair(fgp_fallback=0.15)
    n_full, since, fired = P.O.n_active, 0, 0
    for it in range(cfg["iters"]):
        b = gi.next_batch(S, cfg)
        so = P.O.apply(b)
        assert so[0] == 0
        since += len(b)
        so_st, sto = P.O.refine()
        due = since * 1_000_000 >= 150_000 * n_full
        if due:
            assert P.O.repartition() == 0
            n_full, since = P.O.n_active, 0
            fired += 1
        sg, stg, bad = P.G.step(b)
        assert stg["repartitioned"] == int(due), it
        if not due:
            assert stg["cut"] == sto["cut"]
        P.compare_state(f"it{it}")
    assert 4 <= fired <= 8
