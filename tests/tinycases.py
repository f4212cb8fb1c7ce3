"""Seeded tiny random graphs + valid modifier batches for the brute-force pins
(pure Python; no method arithmetic)."""
from __future__ import annotations

import random

import numpy as np


def random_graph(rng: random.Random, n: int, p: float, weighted: bool):
    edges = {}
    for u in range(n):
        for v in range(u + 1, n):
            if rng.random() < p:
                edges[(u, v)] = rng.randint(1, 3) if weighted else 1
    adj = {u: {} for u in range(n)}
    for (u, v), w in edges.items():
        adj[u][v] = w
        adj[v][u] = w
    xadj = [0]
    adjncy, adjwgt = [], []
    for u in range(n):
        for x in sorted(adj[u]):
            adjncy.append(x)
            adjwgt.append(adj[u][x])
        xadj.append(len(adjncy))
    vw = [rng.randint(1, 3) if weighted else 1 for _ in range(n)]
    return (np.array(xadj, np.int64), np.array(adjncy, np.int32), np.array(adjwgt, np.int32),
            np.array(vw, np.int32), adj)


def random_batch(rng: random.Random, adj, active, weighted: bool, max_ops: int = 6):
    """A valid batch (S1 rules) against the given state."""
    n = len(active)
    live = [u for u in range(n) if active[u]]
    batch = []
    dels = set(rng.sample(live, min(len(live) // 4, rng.randint(0, 2)))) if live else set()
    for u in sorted(dels):
        batch.append([1, u, 0, 0])
    used = set()
    edges = [(u, v) for u in live for v in adj[u] if u < v and u not in dels and v not in dels]
    rng.shuffle(edges)
    for (u, v) in edges[: rng.randint(0, 2)]:
        batch.append([0, u, v, 0])
        used.add((u, v))
    nvi = rng.randint(0, 2)
    for _ in range(nvi):
        batch.append([2, 0, 0, rng.randint(1, 3) if weighted else 1])
    cands = [u for u in live if u not in dels] + list(range(n, n + nvi))
    for _ in range(rng.randint(0, max_ops)):
        if len(cands) < 2:
            break
        u, v = rng.sample(cands, 2)
        a, b = min(u, v), max(u, v)
        if (a, b) in used or (a < n and b < n and b in adj[a]):
            continue
        used.add((a, b))
        batch.append([3, u, v, rng.randint(1, 3) if weighted else 1])
    rng.shuffle(batch)
    # vertex insertions keep their relative order (it defines the new IDs);
    # shuffling moved them, so renumber: the j-th VI in the list is ID n + j.
    return np.array(batch, np.int32).reshape(-1, 4)
