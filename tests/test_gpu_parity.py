"""GPU parity: the CUDA path (C ABI) vs the CPU oracle, bit-exact.

Covers the worked examples, tiny random graphs (weighted and unit), invalid
batches (atomic rejection with the same first index), the BASELINE configs C1
(all 20 iterations), C2 (1M vertices, full-size, 100 iterations; 1000 under
the `slow` marker), C3-style k / batch sweeps, C5-style forced restoration,
batch-order invariance, multi-apply accumulation and edge cases.
"""
import functools
import json
import os
import random

import numpy as np
import pytest

import igk_inputs as gi
from tests.parity import COMMON, Pair, run_stream
from tests.tinycases import random_batch, random_graph

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden", "examples.json")


def _csr(n, edges):
    adj = {u: set() for u in range(n)}
    for u, v in edges:
        adj[u].add(v)
        adj[v].add(u)
    xadj, a = [0], []
    for u in range(n):
        a += sorted(adj[u])
        xadj.append(len(a))
    return np.array(xadj, np.int64), np.array(a, np.int32)


@pytest.mark.parametrize("ex", json.load(open(GOLD))["examples"], ids=lambda e: e["name"])
def test_worked_examples(ex):
    xadj, adj = _csr(ex["n"], ex["edges"])
    P = Pair(xadj, adj, ex["k"], ex["eps"], np.array(ex["part0"], np.int32))
    assert P.apply(np.array(ex["batch"], np.int32)) == 0
    P.compare_state("after apply", full_csr=True)
    sto, stg = P.refine()
    assert list(P.G.partition()) == ex["final_part"]
    assert stg["cut"] == ex["final_cut"] and stg["rounds"] == ex["rounds"]
    P.compare_state("after refine", full_csr=True)


def _tiny(seed):
    rng = random.Random(seed)
    n = rng.randint(3, 40)
    k = rng.choice([2, 3, 4, 7])
    weighted = rng.random() < 0.4
    eps = rng.choice([0.03, 0.1, 0.5, 1.0])
    xadj, adjncy, adjwgt, vwgt, adj = random_graph(rng, n, rng.choice([0.1, 0.2, 0.4]), weighted)
    part0 = np.array([rng.randrange(k) for _ in range(n)], np.int32)
    P = Pair(xadj, adjncy, k, eps, part0, vwgt if weighted else None, adjwgt if weighted else None)
    P.refine("settle")
    P.compare_state("settle", full_csr=True)
    for it in range(4):
        xa, aj, aw = P.O.export_csr()
        part = P.O.partition()
        cur = {u: {int(aj[j]): int(aw[j]) for j in range(xa[u], xa[u + 1])} for u in range(len(part))}
        active = {u: part[u] != -1 for u in range(len(part))}
        b = random_batch(rng, cur, active, weighted, max_ops=10)
        assert P.apply(b, f"seed{seed} it{it}") == 0
        P.compare_state(f"seed{seed} it{it} apply", full_csr=True)
        P.refine(f"seed{seed} it{it}")
        P.compare_state(f"seed{seed} it{it} refine", full_csr=True)


@pytest.mark.parametrize("seed", range(60))
def test_tiny_random(seed):
    _tiny(seed)


def test_invalid_batches_atomic():
    xadj, adj = _csr(6, [(0, 1), (1, 2), (3, 4), (4, 5)])
    part0 = np.array([0, 0, 0, 1, 1, 1], np.int32)
    bad = [[[0, 0, 2, 0]], [[3, 0, 1, 1]], [[3, 2, 2, 1]], [[1, 7, 0, 0]], [[1, 2, 0, 0], [1, 2, 0, 0]],
           [[3, 0, 3, 1], [3, 3, 0, 1]], [[3, 0, 3, 1], [0, 3, 0, 0]], [[1, 1, 0, 0], [0, 0, 1, 0]],
           [[1, 4, 0, 0], [3, 0, 4, 1]], [[3, 0, 6, 1]], [[2, 0, 0, 1], [3, 0, 7, 1]], [[2, 0, 0, 2]],
           [[3, 0, 3, 2]], [[9, 0, 1, 1]], [[3, 0, 3, 1], [0, 0, 5, 0]], [[3, -1, 3, 1]]]
    P = Pair(xadj, adj, 2, 0.1, part0)
    for b in bad:
        before = (P.G.partition().tobytes(), P.G.export_csr()[1].tobytes())
        st = P.apply(np.array(b, np.int32), str(b))
        assert st == 1, b
        assert (P.G.partition().tobytes(), P.G.export_csr()[1].tobytes()) == before
    # a valid batch still works afterwards
    assert P.apply(np.array([[2, 0, 0, 1], [3, 6, 0, 1], [0, 3, 4, 0]], np.int32)) == 0
    P.refine()
    P.compare_state("after", full_csr=True)


@functools.lru_cache(maxsize=4)
def _cfg_graph(name, idx, n, k, weighted):
    """graph + METIS partition of a BASELINE config, built once per session"""
    cfg = gi.CONFIGS[name]
    g = gi.make_graph(n, cfg["fmax"], gi.graph_seed(idx), weighted=weighted)
    part, _ = gi.metis_partition(g, k)
    return g, part


def _cfg_pair(name, idx, n=None, k=None, weighted=False, check=True, **kw):
    cfg = dict(gi.CONFIGS[name])
    n = n or cfg["n"]
    k = k or (cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0])
    g, part = _cfg_graph(name, idx, n, k, weighted)
    P = Pair(g.xadj, g.adjncy, k, cfg["eps"], part, g.vwgt, g.adjwgt, check=check, **kw)
    return cfg, g, part, P


def test_c1_all_iterations():
    cfg, g, part, P = _cfg_pair("C1", 1)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(1)))
    batches = [gi.next_batch(S, cfg) for _ in range(cfg["iters"])]
    run_stream(P, batches, full_csr_every=5, tag="C1")


def _c2(iters):
    """C2 at full size: partition vector, cut, W_p and the GPU recount
    compared with the oracle after EVERY iteration; the oracle's invariants
    I1-I5 every iteration (I1 on the GPU's maintained cut), I6 every 25th."""
    cfg, g, part, P = _cfg_pair("C2", 2, check=False, struct_every=25)
    P.refine("settle")
    P.compare_state("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(2)))
    for it in range(iters):
        b = gi.next_batch(S, cfg)
        assert P.apply(b, f"C2 it{it}") == 0
        P.refine(f"C2 it{it}")
        P.compare_state(f"C2 it{it}")
    P.compare_state("C2 end", full_csr=True)


def test_c2_full_size_100_iterations():
    _c2(100)


@pytest.mark.slow
def test_c2_full_size_1000_iterations():
    _c2(1000)


@pytest.mark.parametrize("k", [2, 8, 32, 64])
def test_c3_full_size_k_sweep(k):
    """C3 at full size (1M vertices) for every k of the config, at both ends
    of its batch sweep (0.1% and 10% modified vertices per iteration):
    partitions, cuts, W_p and stats bit-exact after every iteration."""
    cfg, g, part, P = _cfg_pair("C3", 3, k=k, check=False, struct_every=3)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(3)) + k)
    for it, frac in enumerate([0.001, 0.001, 0.001, 0.10, 0.10, 0.10]):
        b = S.next(gi.MODE_MIX, frac)
        assert P.apply(b, f"k{k} it{it}") == 0
        P.refine(f"k{k} it{it}")
        P.compare_state(f"k{k} it{it}")


def test_weighted_mixed_stream():
    cfg, g, part, P = _cfg_pair("C1", 6, n=20_000, k=8, weighted=True)
    P.refine("settle")
    P.compare_state("settle")
    S = gi.Stream(g, 99, weighted=True)
    for it in range(10):
        b = S.next(gi.MODE_MIX, 0.02)
        assert P.apply(b, f"w it{it}") == 0
        P.refine(f"w it{it}")
        P.compare_state(f"w it{it}", full_csr=(it % 3 == 0))


def test_adversarial_restoration():
    n, k = 40_000, 8
    g = gi.make_graph(n, 1000, gi.graph_seed(5))
    part, _ = gi.metis_partition(g, k)
    P = Pair(g.xadj, g.adjncy, k, 0.03, part)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(5)), region0=(part == 0).astype(np.int32))
    ev = 0
    for it in range(12):
        b = S.next(gi.MODE_ADVERSARIAL, 0.0, n // 100, n // 200, 0, 0)
        assert P.apply(b, f"adv it{it}") == 0
        sto, stg = P.refine(f"adv it{it}")
        ev += stg["evicted"]
        P.compare_state(f"adv it{it}")
    assert ev > 0


def test_batch_permutation_invariance():
    g = gi.make_graph(5000, 64, 17)
    part = gi.block_partition(g.n, 4)
    S = gi.Stream(g, 3)
    b = S.next(gi.MODE_MIX, 0.05)
    res = []
    for perm in range(3):
        bb = b.copy()
        if perm:
            vi = bb[:, 0] == 2
            others = np.nonzero(~vi)[0]
            rng = np.random.default_rng(perm)
            idx = np.arange(len(bb))
            idx[others] = rng.permutation(others)   # vertex insertions keep their order
            bb = bb[idx]
        P = Pair(g.xadj, g.adjncy, 4, 0.03, part)
        assert P.apply(bb) == 0
        P.refine()
        res.append((P.G.partition().tobytes(), P.G.cut()))
    assert res[0] == res[1] == res[2]


def test_multiple_applies_then_one_refine():
    g = gi.make_graph(20_000, 64, 23)
    part, _ = gi.metis_partition(g, 4)
    P = Pair(g.xadj, g.adjncy, 4, 0.03, part)
    P.refine()
    S = gi.Stream(g, 5)
    for it in range(3):
        for j in range(3):
            assert P.apply(S.next(gi.MODE_MIX, 0.01), f"it{it}.{j}") == 0
            P.compare_state(f"it{it}.{j}")
        P.refine(f"it{it}")
        P.compare_state(f"it{it}", full_csr=True)


def test_edge_cases():
    # empty batch, refine without modifiers, imbalanced start, k=254, growth from n=3
    xadj, adj = _csr(3, [(0, 1)])
    P = Pair(xadj, adj, 2, 0.5, np.array([0, 0, 0], np.int32))
    P.refine("imbalanced start")
    P.compare_state("imbalanced start", full_csr=True)
    assert P.apply(np.zeros((0, 4), np.int32)) == 0
    P.refine("empty")
    P.compare_state("empty")
    batch = [[2, 0, 0, 1]] * 50 + [[3, 3 + i, 3 + (i * 7 + 1) % 50, 1] for i in range(50) if i != (i * 7 + 1) % 50]
    seen = set()
    bb = []
    for m in batch:
        key = (min(m[1], m[2]), max(m[1], m[2]))
        if m[0] == 3 and key in seen:
            continue
        seen.add(key)
        bb.append(m)
    assert P.apply(np.array(bb, np.int32)) == 0
    P.refine("growth")
    P.compare_state("growth", full_csr=True)
    g = gi.make_graph(3000, 64, 31)
    part = (np.arange(g.n) % 254).astype(np.int32)
    Q = Pair(g.xadj, g.adjncy, 254, 0.03, part)
    Q.refine("k254")
    S = gi.Stream(g, 1)
    for it in range(3):
        assert Q.apply(S.next(gi.MODE_MIX, 0.05)) == 0
        Q.refine(f"k254 it{it}")
        Q.compare_state(f"k254 it{it}")


@pytest.mark.parametrize("check", [True, False], ids=["check", "notice"])
@pytest.mark.parametrize("split", ["fused", "split"])
def test_fused_step_api(split, check, monkeypatch):
    """igk_step (apply + refine in one call) == oracle; an invalid batch is
    rejected atomically and the refine is skipped.  "split" forces the
    large-batch launch pair (k_apply at full occupancy + k_refine) that
    igk_step uses from kSplitB modifiers on.  "notice" (check mode off) runs
    the fast completion path: the kernel posts its outputs to host-mapped
    memory and the host polls a flag instead of copying + synchronising."""
    if split == "split":
        monkeypatch.setenv("IGK_SPLIT_B", "1")  # read when the handle is created
    cfg, g, part, P = _cfg_pair("C1", 1, check=check)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(1)) + 1)
    for it in range(8):
        b = gi.next_batch(S, cfg)
        assert P.O.apply(b)[0] == 0
        pre = P.O.partition()
        so, sto = P.O.refine()
        sg, stg, bad = P.G.step(b)
        assert sg == so and bad == -1
        assert all(sto[f] == stg[f] for f in COMMON)
        P.invariants(stg["cut"], f"step it{it}")
        P.check_delta(pre, f"step it{it}")
        P.compare_state(f"step it{it}")
        if it == 3:
            before = (P.G.partition().tobytes(), P.G.cut())
            bad_batch = np.array([[0, 0, 0, 0]], np.int32)  # self loop -> invalid
            sg, stg, bad = P.G.step(bad_batch)
            assert sg == 1 and bad == 0
            assert (P.G.partition().tobytes(), P.G.cut()) == before


def test_c4_full_size_10m():
    """BASELINE C4 at full size (10M vertices, heavy fanout <= 1e4, k=16, 5%
    modified per iteration), ALL 20 iterations: partition vectors, cuts, part
    weights, stats and the GPU recount bit-exact after every iteration;
    invariants I1-I5 every iteration, I6 every 5th."""
    cfg, g, part, P = _cfg_pair("C4", 4, check=False, struct_every=5)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(4)))
    for it in range(cfg["iters"]):
        b = gi.next_batch(S, cfg)
        assert P.apply(b, f"C4 it{it}") == 0
        P.refine(f"C4 it{it}")
        P.compare_state(f"C4 it{it}")


def test_c4_full_size_step_split_launch():
    """C4 through igk_step: its ~280K-modifier batches take the split launch
    (k_apply at full occupancy, then k_refine without a host round trip);
    bit-exact with the oracle for 3 iterations."""
    cfg, g, part, P = _cfg_pair("C4", 4, check=False, struct_every=0)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(4)))
    for it in range(3):
        b = gi.next_batch(S, cfg)
        assert len(b) >= 131072
        assert P.O.apply(b)[0] == 0
        pre = P.O.partition()
        so, sto = P.O.refine()
        sg, stg, bad = P.G.step(b)
        assert sg == so and bad == -1
        diff = {f: (sto[f], stg[f]) for f in COMMON if sto[f] != stg[f]}
        assert not diff, diff
        P.invariants(stg["cut"], f"C4 step it{it}")
        P.check_delta(pre, f"C4 step it{it}")
        P.compare_state(f"C4 step it{it}")


def test_c5_full_size_adversarial():
    """BASELINE C5 at full size (4M vertices, k=8), ALL 21 iterations:
    deletions concentrated in one region; after warm-up the restoration (R3)
    fires every iteration; everything compared after every iteration."""
    cfg, g, part, P = _cfg_pair("C5", 5, check=False, struct_every=7)
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(5)), region0=(part == 0).astype(np.int32))
    evicted = []
    for it in range(cfg["iters"]):
        b = gi.next_batch(S, cfg)
        assert P.apply(b, f"C5 it{it}") == 0
        sto, stg = P.refine(f"C5 it{it}")
        evicted.append(stg["evicted"])
        P.compare_state(f"C5 it{it}")
    assert sum(e > 0 for e in evicted) >= 10, evicted


def _hub_graph(seed, n=12_000, hubs=6, leaves=(1100, 3000)):
    """Sparse random graph plus star hubs of degree > 1024 whose leaves sit
    mostly in other parts, so hubs enter A, C1, N and the rounds."""
    rng = np.random.default_rng(seed)
    edges = set()
    for u in range(n):
        for v in rng.integers(max(0, u - 40), min(n, u + 40), size=2):
            if u != v:
                edges.add((min(u, int(v)), max(u, int(v))))
    hub_ids = rng.choice(n, size=hubs, replace=False)
    for h in hub_ids:
        for v in rng.choice(n, size=int(rng.integers(*leaves)), replace=False):
            if v != h:
                edges.add((min(int(h), int(v)), max(int(h), int(v))))
    xadj, adj = _csr(n, sorted(edges))
    return xadj, adj, hub_ids


def test_hub_cta_paths():
    k = 4
    xadj, adj, hubs = _hub_graph(7)
    n = len(xadj) - 1
    part = gi.block_partition(n, k)
    for i, h in enumerate(hubs):  # hubs start in a part where few of their leaves are
        part[h] = (part[h] + 1 + i) % k
    P = Pair(xadj, adj, k, 0.05, part)
    P.refine("settle")
    P.compare_state("settle")
    g = gi.Graph(*P.O.export_csr()[:2], None, None)
    rng = np.random.default_rng(3)
    for it in range(6):
        xa, aj, _ = P.O.export_csr()
        cur = P.O.partition()
        live = np.nonzero(cur >= 0)[0]
        batch, used = [], set()
        for h in hubs:  # touch every hub: new edges to random live vertices
            if cur[h] < 0:
                continue
            nb = set(aj[xa[h]:xa[h + 1]].tolist())
            for v in rng.choice(live, size=4, replace=False):
                key = (min(int(h), int(v)), max(int(h), int(v)))
                if v != h and int(v) not in nb and key not in used:
                    used.add(key)
                    batch.append([3, int(h), int(v), 1])
            # and delete one existing hub edge
            if xa[h + 1] > xa[h]:
                v = int(aj[xa[h] + it])
                key = (min(int(h), v), max(int(h), v))
                if key not in used:
                    used.add(key)
                    batch.append([0, int(h), v, 0])
        # a couple of vertex insertions attached to hubs (pseudo neighbours of hubs)
        base = len(cur)
        for j in range(3):
            batch.append([2, 0, 0, 1])
            batch.append([3, base + j, int(hubs[j % len(hubs)]), 1])
        b = np.array(batch, np.int32)
        assert P.apply(b, f"hub it{it}") == 0
        sto, stg = P.refine(f"hub it{it}")
        P.compare_state(f"hub it{it}", full_csr=(it % 2 == 0))
    # a hub deletion
    assert P.apply(np.array([[1, int(hubs[0]), 0, 0]], np.int32), "hub delete") == 0
    P.refine("hub delete")
    P.compare_state("hub delete", full_csr=True)


def test_store_maintenance_growth_and_compaction():
    """Store maintenance (NEXT-4): a store created with almost no
    spare vertex IDs or slab slots must grow / compact itself transparently
    (capacity failures are detected before any mutation, then the batch is
    re-run) and stay bit-exact with the oracle, through both the two-call and
    the fused-step entry points and an explicit igk_compact."""
    cfg = dict(gi.CONFIGS["C1"])
    k = cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0]
    g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(1))
    part, _ = gi.metis_partition(g, k)
    deg = np.diff(g.xadj)
    used = int((((deg + np.maximum(2, deg // 4)) + 3) & ~3).sum())
    P = Pair(g.xadj, g.adjncy, k, cfg["eps"], part, g.vwgt, g.adjwgt, check=True,
             max_vertices=cfg["n"] + 8, max_slots=used + 64)
    cap0 = P.G.store_stats()["slab_cap"]
    P.refine("settle")
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(1)))
    for it in range(cfg["iters"]):
        b = gi.next_batch(S, cfg)
        if it % 2 == 0:
            assert P.apply(b, f"it{it}") == 0
            P.refine(f"it{it}")
        else:
            assert P.O.apply(b)[0] == 0
            so, sto = P.O.refine()
            sg, stg, bad = P.G.step(b)
            assert sg == so == 0 and bad == -1
            assert all(sto[f] == stg[f] for f in COMMON)
            P.invariants(stg["cut"], f"it{it}")
        P.compare_state(f"it{it}", full_csr=(it % 5 == 4))
        if it == 10:
            P.G.compact()
            P.compare_state("after explicit compact", full_csr=True)
    ss = P.G.store_stats()
    assert ss["n_total"] > cfg["n"] + 8     # vertex arrays grew
    assert ss["slab_cap"] > cap0            # the slab was compacted into a larger one
    assert ss["slab_top"] <= ss["slab_cap"]
