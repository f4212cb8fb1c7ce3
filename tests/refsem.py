"""Brute-force, tiny-input restatement of each IGK-SEM v1 step, used ONLY to
pin the oracle (tests/test_oracle_pins.py).  Pure Python on dict/set graphs,
O(k^n) enumeration where an optimum is needed.  It shares no code with
oracle/ (C) or the CUDA path; every step is recomputed from the paper's
definitions (Alg. 3, Alg. 4, Fig. 5) without reusing the
oracle's running sums or sort order.
"""
from __future__ import annotations

import itertools
from fractions import Fraction

PSI = -2  # pending (pseudo) label as returned by partition()
DEL = -1


def csr_to_adj(xadj, adjncy, adjwgt=None):
    n = len(xadj) - 1
    adj = {u: {} for u in range(n)}
    for u in range(n):
        for j in range(int(xadj[u]), int(xadj[u + 1])):
            adj[u][int(adjncy[j])] = 1 if adjwgt is None else int(adjwgt[j])
    return adj


def cap_exact(W: int, eps: float, k: int) -> int:
    """P:52 with e = round(eps * 1e6) ppm, in exact rationals (reading Q4)."""
    e = Fraction(round(eps * 1_000_000), 1_000_000)
    return max(int((W * (1 + e)) / k // 1), -(-W // k))


def cut_of(adj, part):
    """sum of W_e over edges whose (placed) endpoints differ."""
    c = 0
    for u, nb in adj.items():
        for x, w in nb.items():
            if u < x and part[u] >= 0 and part[x] >= 0 and part[u] != part[x]:
                c += w
    return c


def apply_batch(adj, active, vw, batch, vw_unit=True):
    """S1 set semantics on an edge-set model.  Returns (adj', active', vw', A, inserted_ids)."""
    adj = {u: dict(nb) for u, nb in adj.items()}
    active = dict(active)
    vw = dict(vw)
    n = len(active)
    A = set()
    ins = []
    for kd, u, v, w in batch:
        if kd == 0:
            del adj[u][v]
            del adj[v][u]
            A |= {u, v}
    for kd, u, v, w in batch:
        if kd == 1:
            for x in list(adj[u]):
                del adj[x][u]
                A.add(x)
            adj[u] = {}
            active[u] = False
    for kd, u, v, w in batch:
        if kd == 2:
            nid = n + len(ins)
            ins.append(nid)
            adj[nid] = {}
            active[nid] = True
            vw[nid] = w
    for kd, u, v, w in batch:
        if kd == 3:
            adj[u][v] = w
            adj[v][u] = w
            A |= {u, v}
    A = {u for u in A if active[u]}
    return adj, active, vw, A, ins


def int_ext(adj, part, u):
    i = sum(w for x, w in adj[u].items() if part[x] == part[u])
    e = sum(w for x, w in adj[u].items() if part[x] != part[u])
    return i, e


def part_weights(part, vw, active, k):
    Wp = [0] * k
    for u, p in part.items():
        if active[u] and p >= 0:
            Wp[p] += vw[u]
    return Wp


def replay_refine(adj, active, vw, part, A, k, eps):
    """Recompute R1-R4 by brute force.  Returns a trace dict."""
    part = dict(part)
    W = sum(vw[u] for u in active if active[u])
    c = cap_exact(W, eps, k)
    # R1 (Alg. 3 L8-24): u in A, placed, ext > int, on sigma1
    s1 = dict(part)
    C1 = {u for u in A if s1[u] >= 0 and (lambda ie: ie[1] > ie[0])(int_ext(adj, s1, u))}
    for u in C1:
        part[u] = PSI
    # R2: placed neighbours of pseudo vertices, same filter on sigma2
    s2 = dict(part)
    N = {x for u in adj if active[u] and s2[u] == PSI for x in adj[u] if s2[x] >= 0}
    C2 = {x for x in N if (lambda ie: ie[1] > ie[0])(int_ext(adj, s2, x))}
    for x in C2:
        part[x] = PSI
    # R3: shortest prefix by (int - ext, id) with weight >= W_i - c, each part
    s3 = dict(part)
    Wp = part_weights(s3, vw, active, k)
    R3 = set()
    for i in range(k):
        if Wp[i] <= c:
            continue
        need = Wp[i] - c
        members = sorted((int_ext(adj, s3, x)[0] - int_ext(adj, s3, x)[1], x)
                         for x in adj if active[x] and s3[x] == i)
        # brute force over prefix lengths: the shortest one that reaches need
        for ell in range(len(members) + 1):
            if sum(vw[x] for _, x in members[:ell]) >= need:
                R3 |= {x for _, x in members[:ell]}
                break
    for x in R3:
        part[x] = PSI
    # R4 rounds (Alg. 4)
    rounds = []
    imbalanced = False
    while any(active[u] and part[u] == PSI for u in adj):
        Wr = part_weights(part, vw, active, k)
        psi = [u for u in sorted(adj) if active[u] and part[u] == PSI]
        S = [u for u in psi if not any(part[x] == PSI and x < u for x in adj[u])]
        moves = []
        for u in S:
            conn = [sum(w for x, w in adj[u].items() if part[x] == p) for p in range(k)]
            E = [p for p in range(k) if Wr[p] + vw[u] <= c]
            if not E:
                E = [min(range(k), key=lambda p: (Wr[p], p))]
                imbalanced = True
            best = max(E, key=lambda p: (conn[p], -Wr[p], -p))
            moves.append((u, best, conn[best]))
        moves.sort(key=lambda m: (-m[2], m[0]))
        # longest prefix such that every part stays within c (Fig. 5),
        # recomputing each prefix's part weights from scratch
        L = 0
        for ell in range(len(moves) + 1):
            Wt = list(Wr)
            for (u, p, g) in moves[:ell]:
                Wt[p] += vw[u]
            if all(Wt[p] <= c for p in range(k)):
                L = ell
            else:
                break
        if L == 0:
            L = 1
            imbalanced = True
        for (u, p, g) in moves[:L]:
            part[u] = p
        rounds.append((moves, L))
    return dict(C1=C1, C2=C2, R3=R3, rounds=rounds, part=part, cap=c, N=N, imbalanced=imbalanced)


def brute_force_opt(adj, active, vw, k, c):
    """Minimum cut over all k-way partitions of the active vertices with every
    part weight <= c (exhaustive; tiny n only)."""
    verts = [u for u in sorted(adj) if active[u]]
    best = None
    for assign in itertools.product(range(k), repeat=len(verts)):
        Wp = [0] * k
        for u, p in zip(verts, assign):
            Wp[p] += vw[u]
        if max(Wp) > c:
            continue
        part = {u: -1 for u in adj}
        part.update(dict(zip(verts, assign)))
        cut = cut_of(adj, part)
        if best is None or cut < best:
            best = cut
    return best
