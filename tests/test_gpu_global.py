"""GPU parity of NEXT-1 global boundary refinement (igk_refine_global; P:140,
SURVEY 8(f)) against the oracle's ora_refine_global, bit-exact: the worked
example, tiny random graphs (weighted and unit, with pending pseudo vertices
present when the call is made), C1 with a global pass every 5 iterations, the
hub (degree > 1024) paths of the boundary scan, and full-size C2 and C4."""
import json
import os
import random

import numpy as np
import pytest

import igk_inputs as gi
from tests.parity import Pair
from tests.test_gpu_parity import _cfg_pair, _csr, _hub_graph
from tests.tinycases import random_batch, random_graph

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden", "global_examples.json")


@pytest.mark.parametrize("ex", json.load(open(GOLD))["examples"], ids=lambda e: e["name"])
def test_global_worked_example(ex):
    xadj, adj = _csr(ex["n"], ex["edges"])
    P = Pair(xadj, adj, ex["k"], ex["eps"], np.array(ex["part0"], np.int32))
    P.refine("plain")
    sto, stg = P.refine_global("global")
    assert list(P.G.partition()) == ex["final_part"] and stg["cut"] == ex["final_cut"]
    P.compare_state("after global", full_csr=True)


@pytest.mark.parametrize("seed", range(40))
def test_global_tiny_random(seed):
    rng = random.Random(5000 + seed)
    n = rng.randint(3, 60)
    k = rng.choice([2, 3, 4, 7])
    weighted = rng.random() < 0.4
    eps = rng.choice([0.03, 0.1, 0.5, 1.0])
    xadj, adjncy, adjwgt, vwgt, adj = random_graph(rng, n, rng.choice([0.05, 0.1, 0.3]), weighted)
    part0 = np.array([rng.randrange(k) for _ in range(n)], np.int32)
    P = Pair(xadj, adjncy, k, eps, part0, vwgt if weighted else None, adjwgt if weighted else None)
    P.refine_global("initial global")
    P.compare_state("initial global", full_csr=True)
    for it in range(4):
        xa, aj, aw = P.O.export_csr()
        part = P.O.partition()
        cur = {u: {int(aj[j]): int(aw[j]) for j in range(xa[u], xa[u + 1])} for u in range(len(part))}
        active = {u: part[u] != -1 for u in range(len(part))}
        assert P.apply(random_batch(rng, cur, active, weighted, max_ops=10), f"s{seed} it{it}") == 0
        # global refine right after an apply: pseudo vertices are pending (external to the scan)
        (P.refine_global if it % 2 == 0 else P.refine)(f"s{seed} it{it}")
        P.compare_state(f"s{seed} it{it}", full_csr=(it == 3))


def test_global_c1_every_5_iterations():
    cfg, g, part, P = _cfg_pair("C1", 1)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(1)))
    for it in range(cfg["iters"]):
        assert P.apply(gi.next_batch(S, cfg), f"C1 it{it}") == 0
        P.refine(f"C1 it{it}")
        if it % 5 == 4:
            P.refine_global(f"C1 it{it} global")
        P.compare_state(f"C1 it{it}")


def test_global_hub_paths():
    k = 4
    xadj, adj, hubs = _hub_graph(11)
    n = len(xadj) - 1
    part = gi.block_partition(n, k)
    for i, h in enumerate(hubs):
        part[h] = (part[h] + 1 + i) % k
    P = Pair(xadj, adj, k, 0.05, part)
    sto, stg = P.refine_global("hubs global")
    assert stg["affected"] >= len(hubs)
    P.compare_state("hubs global", full_csr=True)
    P.refine_global("hubs global 2")
    P.compare_state("hubs global 2")


@pytest.mark.parametrize("name,idx,iters", [("C2", 2, 12), ("C4", 4, 2)])
def test_global_full_size(name, idx, iters):
    cfg, g, part, P = _cfg_pair(name, idx, check=False)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(idx)))
    for it in range(iters):
        assert P.apply(gi.next_batch(S, cfg), f"{name} it{it}") == 0
        P.refine(f"{name} it{it}")
    sto, stg = P.refine_global(f"{name} global")
    assert stg["affected"] > 0.01 * g.n  # the boundary of a METIS partition is a few % of n
    P.compare_state(f"{name} global")
