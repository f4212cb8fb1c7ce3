"""Pins the oracle's NEXT-1 global boundary refinement (ora_refine_global,
SURVEY 8(f) NEXT-1: G-kway "refines all vertices on the partition
boundary (i.e., vertices with adj_ext != 0)") to things other than itself:
  * a hand-worked example (tests/golden/global_examples.json),
  * the brute-force replay of tests/refsem.py with A := A u B, where the
    boundary B is recomputed here from the exported graph (reading B1),
  * an equivalence through a different code path: after a refine (Psi empty)
    the boundary is exactly the set of cut-edge endpoints, so deleting every
    cut edge and inserting it back (two ordinary applies, same graph) followed
    by refine() must give the same result as refine_global().
CPU only."""
import json
import os
import random

import numpy as np
import pytest

import oracle
from tests import refsem
from tests.test_oracle_pins import _csr, _state_from_oracle
from tests.tinycases import random_batch, random_graph

GOLD = os.path.join(os.path.dirname(__file__), "golden", "global_examples.json")


def _boundary(adj, active, part):
    """B = placed active vertices with adj_ext != 0 (a pseudo neighbour is
    external, reading Q13) -- written out from the definition."""
    return {u for u in adj if active[u] and part[u] >= 0 and any(part[x] != part[u] for x in adj[u])}


@pytest.mark.parametrize("ex", json.load(open(GOLD))["examples"], ids=lambda e: e["name"])
def test_global_worked_example(ex):
    xadj, adj = _csr(ex["n"], ex["edges"])
    O = oracle.Oracle(xadj, adj, ex["k"], ex["eps"], np.array(ex["part0"], np.int32))
    s, st = O.refine()  # A is empty: an ordinary refine changes nothing
    assert list(O.partition()) == ex["part0"] and st["rounds"] == 0
    s, st = O.refine_global()
    assert s == 0
    assert st["cap"] == ex["cap"]
    assert st["affected"] == ex["affected"]
    assert st["filtered_in"] == ex["filtered_in"]
    assert st["expanded_in"] == ex["expanded_in"]
    assert st["rounds"] == ex["rounds"]
    assert list(O.partition()) == ex["final_part"]
    assert O.cut() == st["cut"] == ex["final_cut"]
    assert O.check_invariants() is None


def _global_case(seed):
    rng = random.Random(seed)
    n = rng.randint(3, 10)
    k = rng.choice([2, 2, 3])
    weighted = rng.random() < 0.3
    eps = rng.choice([0.03, 0.1, 0.5, 1.0])
    xadj, adjncy, adjwgt, vwgt, _ = random_graph(rng, n, rng.choice([0.2, 0.35, 0.5]), weighted)
    part0 = np.array([rng.randrange(k) for _ in range(n)], np.int32)
    O = oracle.Oracle(xadj, adjncy, k, eps, part0, vwgt if weighted else None, adjwgt if weighted else None)
    vw = {u: int(vwgt[u]) if weighted else 1 for u in range(n)}
    for it in range(3):
        adj0, active0, _ = _state_from_oracle(O)
        batch = random_batch(rng, adj0, active0, weighted)
        assert O.apply(batch)[0] == 0
        adj1, active1, vw1, A, ins = refsem.apply_batch(adj0, active0, vw, batch.tolist())
        vw = vw1
        _, _, sigma = _state_from_oracle(O)
        B = _boundary(adj1, active1, sigma)
        s, st = O.refine_global()
        ref = refsem.replay_refine(adj1, active1, vw, sigma, set(A) | B, k, eps)
        c1, c2, r3 = O.trace_sets()
        assert set(np.nonzero(c1)[0]) == ref["C1"], (seed, it)
        assert set(np.nonzero(c2)[0]) == ref["C2"], (seed, it)
        assert set(np.nonzero(r3)[0]) == ref["R3"], (seed, it)
        part = O.partition()
        assert {u: int(part[u]) for u in range(len(part))} == \
            {u: (ref["part"][u] if active1[u] else -1) for u in ref["part"]}
        assert bool(st["imbalanced"]) == ref["imbalanced"]
        assert O.check_invariants() is None


@pytest.mark.parametrize("seed", range(200))
def test_global_replay_tiny_random(seed):
    _global_case(seed)


def _cut_edges(O):
    xa, aj, aw = O.export_csr()
    part = O.partition()
    out = []
    for u in range(len(part)):
        for j in range(xa[u], xa[u + 1]):
            v = int(aj[j])
            if u < v and part[u] != part[v]:
                out.append((u, v, int(aw[j])))
    return out


@pytest.mark.parametrize("seed", range(60))
def test_global_equals_cut_edge_reinsertion(seed):
    rng = random.Random(1000 + seed)
    n = rng.randint(8, 60)
    k = rng.choice([2, 3, 4])
    weighted = rng.random() < 0.3
    xadj, adjncy, adjwgt, vwgt, _ = random_graph(rng, n, rng.choice([0.08, 0.15, 0.3]), weighted)
    part0 = np.array([rng.randrange(k) for _ in range(n)], np.int32)
    args = (xadj, adjncy, k, 0.1, part0, vwgt if weighted else None, adjwgt if weighted else None)
    Og, Oe = oracle.Oracle(*args), oracle.Oracle(*args)
    Og.refine()
    Oe.refine()
    cuts = _cut_edges(Oe)
    _, stg = Og.refine_global()
    if cuts:
        assert Oe.apply(np.array([[0, u, v, 0] for u, v, _ in cuts], np.int32))[0] == 0
        assert Oe.apply(np.array([[3, u, v, w] for u, v, w in cuts], np.int32))[0] == 0
    _, ste = Oe.refine()
    assert np.array_equal(Og.partition(), Oe.partition())
    for f in ("affected", "filtered_in", "expanded_in", "evicted", "rounds", "moves_applied", "cut"):
        assert stg[f] == ste[f], f


def test_global_on_generated_graph_keeps_invariants_and_never_loses_balance():
    import igk_inputs as gi
    g = gi.make_graph(3000, 64, gi.graph_seed(1))
    part = gi.block_partition(g.n, 4)
    O = oracle.Oracle(g.xadj, g.adjncy, 4, 0.03, part)
    O.refine()
    S = gi.Stream(g, 11)
    for it in range(4):
        assert O.apply(S.next(gi.MODE_MIX, 0.02))[0] == 0
        s, st = (O.refine_global() if it % 2 else O.refine())
        assert s == 0 and O.check_invariants() is None
        assert st["max_part_weight"] <= st["cap"]
