"""Pins the CPU oracle to things other than itself (CPU only, -m "not gpu"):
  * the hand-worked examples in tests/golden/examples.json (Fig. 5 + Ex1-Ex6),
  * the closed form of the balance bound in exact rationals,
  * a brute-force step-by-step replay (tests/refsem.py) of apply (S1), R1 filter,
    R2 expansion, R3 restoration, and every round's selection, best part,
    order and balanced prefix (Alg. 3, Alg. 4, Fig. 5) on tiny random inputs,
  * exhaustive optimum cuts (cut >= OPT; equality on the worked examples),
  * invariants I1-I6, batch-order invariance and invalid-batch atomicity.
"""
import json
import os
import random

import numpy as np
import pytest

import oracle
from tests import refsem
from tests.tinycases import random_batch, random_graph

GOLD = os.path.join(os.path.dirname(__file__), "golden", "examples.json")


def _csr(n, edges):
    adj = {u: set() for u in range(n)}
    for u, v in edges:
        adj[u].add(v)
        adj[v].add(u)
    xadj = [0]
    a = []
    for u in range(n):
        a += sorted(adj[u])
        xadj.append(len(a))
    return np.array(xadj, np.int64), np.array(a, np.int32)


def _examples():
    return json.load(open(GOLD))["examples"]


@pytest.mark.parametrize("ex", _examples(), ids=lambda e: e["name"])
def test_worked_example(ex):
    xadj, adj = _csr(ex["n"], ex["edges"])
    O = oracle.Oracle(xadj, adj, ex["k"], ex["eps"], np.array(ex["part0"], np.int32))
    st, fid, bad = O.apply(np.array(ex["batch"], np.int32))
    assert st == 0 and bad == -1
    s, stats = O.refine()
    assert s == 0
    assert stats["cap"] == ex["cap"]
    assert stats["filtered_in"] == ex["filtered_in"]
    assert stats["expanded_in"] == ex["expanded_in"]
    assert stats["evicted"] == ex["evicted"]
    assert list(O.partition()) == ex["final_part"]
    assert O.cut() == ex["final_cut"] == stats["cut"]
    assert stats["rounds"] == ex["rounds"]
    if "round_sizes" in ex:
        S, L = O.trace_rounds()
        assert [[int(a), int(b)] for a, b in zip(S, L)] == ex["round_sizes"]
    assert O.check_invariants() is None
    # the stated final cut is the exhaustive optimum under the cap
    n = O.n_total
    part = O.partition()
    full = {u: {} for u in range(n)}
    xa, aj, _ = O.export_csr()
    for u in range(n):
        for j in range(xa[u], xa[u + 1]):
            full[u][int(aj[j])] = 1
    active = {u: part[u] != -1 for u in range(n)}
    vw = {u: 1 for u in range(n)}
    assert refsem.brute_force_opt(full, active, vw, ex["k"], ex["cap"]) == ex["final_cut"]


@pytest.mark.parametrize("W,eps,k", [(9, 0.03, 2), (8, 0.03, 2), (11, 0.03, 2), (6, 0.5, 2),
                                     (1_000_000, 0.03, 4), (999_983, 0.03, 64), (1, 0.03, 254),
                                     (2**42, 1.0, 2), (2**42 - 7, 0.001, 253), (133, 0.03, 4),
                                     (134, 0.03, 4), (2133, 0.03, 64), (2134, 0.03, 64),
                                     (10_000_000, 0.0000004, 16)])
def test_cap_closed_form(W, eps, k):
    assert oracle.cap(W, eps, k) == refsem.cap_exact(W, eps, k)


def test_cap_unit_weight_guarantee():
    # balance guarantee: sum W_p <= W - 1 < k c  => some part has room
    for W in range(1, 3000, 7):
        for k in (2, 3, 4, 8, 64):
            c = oracle.cap(W, 0.03, k)
            assert k * c >= W and c >= -(-W // k)


def _state_from_oracle(O, weighted_vw=None):
    n = O.n_total
    xa, aj, aw = O.export_csr()
    adj = {u: {} for u in range(n)}
    for u in range(n):
        for j in range(xa[u], xa[u + 1]):
            adj[u][int(aj[j])] = int(aw[j])
    part = O.partition()
    active = {u: part[u] != -1 for u in range(n)}
    return adj, active, {u: int(part[u]) for u in range(n)}


def _run_case(seed):
    rng = random.Random(seed)
    n = rng.randint(3, 9)
    k = rng.choice([2, 2, 3])
    weighted = rng.random() < 0.3
    eps = rng.choice([0.03, 0.1, 0.5, 1.0])
    xadj, adjncy, adjwgt, vwgt, _ = random_graph(rng, n, rng.choice([0.2, 0.35, 0.5]), weighted)
    part0 = np.array([rng.randrange(k) for _ in range(n)], np.int32)
    O = oracle.Oracle(xadj, adjncy, k, eps, part0, vwgt if weighted else None, adjwgt if weighted else None)
    vw = {u: int(vwgt[u]) if weighted else 1 for u in range(n)}
    for it in range(3):
        adj0, active0, part_pre = _state_from_oracle(O)
        batch = random_batch(rng, adj0, active0, weighted)
        st, fid, bad = O.apply(batch)
        assert st == 0, (seed, it, batch, bad)
        # S1 pinned by an independent edge-set model
        adj1, active1, vw1, A, ins = refsem.apply_batch(adj0, active0, vw, batch.tolist())
        vw = vw1
        adj_o, active_o, sigma1 = _state_from_oracle(O)
        assert adj_o == adj1
        assert active_o == active1
        for u in ins:
            assert sigma1[u] == refsem.PSI
        O_part_before = dict(sigma1)
        s, stats = O.refine()
        ref = refsem.replay_refine(adj1, active1, vw, O_part_before, A, k, eps)
        c1, c2, r3 = O.trace_sets()
        assert set(np.nonzero(c1)[0]) == ref["C1"], (seed, it)
        assert set(np.nonzero(c2)[0]) == ref["C2"], (seed, it)
        assert set(np.nonzero(r3)[0]) == ref["R3"], (seed, it)
        assert stats["cap"] == ref["cap"]
        S, L = O.trace_rounds()
        mv = O.trace_moves()
        assert len(S) == len(ref["rounds"])
        off = 0
        for r, (moves, Lr) in enumerate(ref["rounds"]):
            got = [tuple(int(x) for x in row) for row in mv[off: off + S[r]]]
            assert got == moves, (seed, it, r)
            assert L[r] == Lr
            off += S[r]
        part = O.partition()
        assert {u: int(part[u]) for u in range(len(part))} == {u: (ref["part"][u] if active1[u] else -1) for u in ref["part"]}
        # maintained W_p and W (apply, commits, rounds) == a recount from the labels
        assert list(O.part_weights()) == [sum(vw[u] for u in range(len(part)) if part[u] == p) for p in range(k)]
        assert O.total_weight() == sum(vw[u] for u in range(len(part)) if part[u] >= 0)
        assert O.cut() == stats["cut"] == refsem.cut_of(adj1, {u: int(part[u]) for u in range(len(part))})
        assert bool(stats["imbalanced"]) == ref["imbalanced"]
        assert O.check_invariants() is None
        if not weighted:
            assert stats["imbalanced"] == 0
            assert stats["max_part_weight"] <= stats["cap"]
        nact = sum(active1.values())
        if k ** nact <= 20000 and not stats["imbalanced"]:
            opt = refsem.brute_force_opt(adj1, active1, vw, k, stats["cap"])
            if opt is not None:
                assert stats["cut"] >= opt


@pytest.mark.parametrize("seed", range(400))
def test_replay_tiny_random(seed):
    _run_case(seed)


def test_batch_order_invariance():
    # S1: each phase is a set operation; only the relative order of vertex
    # insertions (which fixes new IDs) matters.
    for seed in range(60):
        rng = random.Random(1000 + seed)
        xadj, adjncy, adjwgt, vwgt, adj = random_graph(rng, 9, 0.35, False)
        part0 = np.array([rng.randrange(2) for _ in range(9)], np.int32)
        batch = random_batch(rng, adj, {u: True for u in range(9)}, False)
        res = []
        for perm in range(3):
            b = batch.copy()
            if perm:
                r2 = random.Random(perm)
                idx = list(range(len(b)))
                r2.shuffle(idx)
                b = b[idx]
            O = oracle.Oracle(xadj, adjncy, 2, 0.1, part0)
            assert O.apply(b)[0] == 0
            s, st = O.refine()
            res.append((tuple(O.partition()), st["cut"]))
        assert res[0] == res[1] == res[2]


def test_invalid_batches_are_atomic():
    xadj, adj = _csr(6, [(0, 1), (1, 2), (3, 4), (4, 5)])
    part0 = np.array([0, 0, 0, 1, 1, 1], np.int32)
    bad_batches = [
        ([[0, 0, 2, 0]], 0),                    # delete a missing edge
        ([[3, 0, 1, 1]], 0),                    # insert an existing edge
        ([[3, 2, 2, 1]], 0),                    # self loop
        ([[1, 7, 0, 0]], 0),                    # delete a missing vertex
        ([[1, 2, 0, 0], [1, 2, 0, 0]], 0),      # vertex deleted twice
        ([[3, 0, 3, 1], [3, 3, 0, 1]], 0),      # same edge twice
        ([[3, 0, 3, 1], [0, 3, 0, 0]], 0),      # insert + delete of one edge
        ([[1, 1, 0, 0], [0, 0, 1, 0]], 1),      # edge delete with a deleted endpoint
        ([[1, 4, 0, 0], [3, 0, 4, 1]], 1),      # insert an edge to a deleted vertex
        ([[3, 0, 6, 1]], 0),                    # new-vertex ID without an insertion
        ([[2, 0, 0, 1], [3, 0, 7, 1]], 1),      # ID beyond the inserted range
        ([[2, 0, 0, 2]], 0),                    # weight on an unweighted handle
        ([[3, 0, 3, 2]], 0),                    # edge weight on an unweighted handle
        ([[9, 0, 1, 1]], 0),                    # unknown kind
        ([[3, 0, 3, 1], [0, 0, 5, 0]], 1),      # second modifier invalid
    ]
    for b, idx in bad_batches:
        O = oracle.Oracle(xadj, adj, 2, 0.1, part0)
        before = (tuple(O.partition()), O.export_csr()[1].tobytes())
        st, fid, bad = O.apply(np.array(b, np.int32))
        assert st == oracle.EINVAL, b
        assert bad == idx, (b, bad)
        assert (tuple(O.partition()), O.export_csr()[1].tobytes()) == before


def test_refine_without_modifiers_is_noop():
    rng = random.Random(5)
    xadj, adjncy, _, _, _ = random_graph(rng, 9, 0.4, False)
    part0 = np.array([0, 0, 0, 0, 1, 1, 1, 1, 1], np.int32)
    O = oracle.Oracle(xadj, adjncy, 2, 0.5, part0)
    s, st = O.refine()
    assert list(O.partition()) == list(part0)
    assert st["rounds"] == 0 and st["evicted"] == 0


def test_imbalanced_initial_partition_is_restored():
    rng = random.Random(6)
    xadj, adjncy, _, _, _ = random_graph(rng, 9, 0.4, False)
    part0 = np.zeros(9, np.int32)
    O = oracle.Oracle(xadj, adjncy, 3, 0.03, part0)
    s, st = O.refine()
    assert s == 0 and st["max_part_weight"] <= st["cap"] == 3
    assert O.check_invariants() is None
