"""Pins of the oracle's invariant checker and of its create-time validation
(CPU only, -m "not gpu").

The invariants are the north_star's ("cut equals a recount; part weights sum
to the total; every part <= (1+eps) W / k; only frontier vertices moved")
plus I5/I6 of SURVEY 8(c) (P:48 graph model, P:52 balance, P:182-188
frontier, P:206 empty pseudo-partition).  A checker that always answers
"fine" -- or one with a plausible slip (I3 inverted, I4 reading the wrong
array, I6 missing one direction) -- must fail here: every test builds a real
state with the oracle, corrupts exactly ONE field through the test-only
hooks, and asserts that ora_check_invariants_ext reports exactly that
invariant (tag "I1".."I6"); the untouched state must pass.

The create-time rejections of ora_create (asymmetric, duplicate, self loop,
out-of-range IDs/weights/parts, bad k/eps, malformed xadj) are checked on
hand-made CSRs, and so is the product's host-side igk_create validation (it
rejects the same inputs before touching the GPU, so this runs on CPU).
"""
import ctypes as C

import numpy as np
import pytest

import igk_inputs as gi
import oracle


def _state(weighted=False):
    """A 3000-vertex oracle after settle + one mixed batch with vertex
    deletions and insertions + refine: some vertices are in the frontier F
    of the last refine, most are not; some IDs are deleted."""
    g = gi.make_graph(3000, 64, 4242, weighted=weighted)
    part = gi.block_partition(g.n, 4)
    O = oracle.Oracle(g.xadj, g.adjncy, 4, 0.03, part, g.vwgt, g.adjwgt)
    O.refine()
    S = gi.Stream(g, 99, weighted=weighted)
    assert O.apply(S.next(gi.MODE_MIX, 0.05))[0] == 0
    O.refine()
    assert O.check_invariants(O.cut()) is None
    return O


def _frontier_flags(O):
    c1, c2, r3 = O.trace_sets()
    n = O.n_total
    part = O.partition()
    # F = every vertex that entered Psi in the last refine: C1, C2, R3 and the
    # inserted ones (IDs beyond the pre-batch range carry their own flag)
    return c1 | c2 | r3, part


def _neighbours(O):
    xa, aj, aw = O.export_csr()
    return xa, aj, aw


def _tag(msg):
    return None if msg is None else msg.split(":")[0]


def test_untouched_state_passes_and_i1_reads_the_reported_cut():
    O = _state()
    assert O.check_invariants() is None
    assert O.check_invariants(O.cut()) is None
    assert _tag(O.check_invariants(O.cut() + 1)) == "I1"
    assert _tag(O.check_invariants(max(O.cut() - 3, 0))) == "I1"


def test_i6_asymmetric_edge():
    O = _state()
    xa, aj, _ = _neighbours(O)
    part = O.partition()
    live = np.nonzero(part >= 0)[0]
    u = int(live[10])
    nb = set(aj[xa[u]:xa[u + 1]].tolist())
    x = next(int(v) for v in live[::-1] if int(v) != u and int(v) not in nb)
    O.debug_add_half_edge(u, x, 1)          # u -> x without x -> u
    assert _tag(O.check_invariants()) == "I6"
    assert "asymmetric" in O.check_invariants()
    assert O.check_invariants(structure=False) is None   # I6 skipped on request only


def test_i6_unequal_weights_both_ways():
    O = _state(weighted=True)
    xa, aj, aw = _neighbours(O)
    u = next(v for v in range(O.n_total) if xa[v + 1] > xa[v])
    x = int(aj[xa[u]])
    O.debug_set_edge_weight(u, x, int(aw[xa[u]]) % 4 + 1)  # w_ux != w_xu
    assert "asymmetric" in O.check_invariants()


def test_i6_duplicate_edge():
    O = _state()
    xa, aj, _ = _neighbours(O)
    u = next(v for v in range(O.n_total) if xa[v + 1] > xa[v])
    x = int(aj[xa[u]])
    O.debug_add_half_edge(u, x, 1)          # both directions twice: symmetric, not simple
    O.debug_add_half_edge(x, u, 1)
    assert "duplicate" in O.check_invariants()


def test_i6_self_loop_and_inactive_endpoint():
    O = _state()
    part = O.partition()
    live = np.nonzero(part >= 0)[0]
    dead = np.nonzero(part == -1)[0]
    assert len(dead) > 0
    O.debug_add_half_edge(int(live[5]), int(live[5]), 1)
    assert "bad neighbour" in O.check_invariants()
    O2 = _state()
    O2.debug_add_half_edge(int(live[5]), int(dead[0]), 1)   # edge into a deleted vertex
    assert _tag(O2.check_invariants()) == "I6"
    O3 = _state()
    O3.debug_add_half_edge(int(dead[0]), int(live[5]), 1)   # a deleted vertex keeps an edge
    assert "deleted" in O3.check_invariants()


def test_i5_pending_vertex_left():
    O = _state()
    part = O.partition()
    v = int(np.nonzero(part >= 0)[0][7])
    O.debug_set_part(v, -1)                 # psi after the refine
    assert _tag(O.check_invariants()) == "I5"


def test_i2_part_weight_and_total_weight():
    O = _state()
    wp = O.part_weights()
    O.debug_set_part_weight(0, wp[0] + 1)   # W_0 off by one, W_1 compensates: sum still = W
    O.debug_set_part_weight(1, wp[1] - 1)
    assert O.check_invariants().startswith("I2: W_0")
    O2 = _state()
    O2.debug_set_total_weight(O2.total_weight() + 1)
    assert O2.check_invariants().startswith("I2: W mismatch")


def test_i3_overweight_part():
    O = _state()
    part = O.partition()
    wp = O.part_weights()
    a, b = 0, 1
    movers = np.nonzero(part == a)[0][: 400]   # 400 unit vertices a -> b: b far above cap
    for v in movers:
        O.debug_set_part(int(v), b)
        O.debug_set_frontier(int(v), 1)     # they count as frontier: I4 must stay quiet
    O.debug_set_part_weight(a, wp[a] - len(movers))
    O.debug_set_part_weight(b, wp[b] + len(movers))
    assert wp[b] + len(movers) > O.cap()
    assert _tag(O.check_invariants()) == "I3"


def test_i4_non_frontier_vertex_moved():
    O = _state()
    F, part = _frontier_flags(O)
    n0 = len(F)
    cand = [v for v in range(3000) if part[v] >= 0 and not F[v]]  # pre-batch IDs (inserted ones have no previous part)
    u = next(v for v in cand if part[v] == 0)
    x = next(v for v in cand if part[v] == 1)
    O.debug_set_part(u, 1)                  # swap two non-frontier vertices: W_p unchanged
    O.debug_set_part(x, 0)
    assert _tag(O.check_invariants()) == "I4"


def test_i4_frontier_vertex_may_move():
    # the converse: a vertex of F changing part (weights kept consistent and
    # within the cap) is legal -- a checker that flags every label change fails
    O = _state()
    F, part = _frontier_flags(O)
    wp = O.part_weights()
    c = O.cap()
    moved = False
    for v in np.nonzero(F)[0]:
        a = int(part[v])
        b = next((p for p in range(4) if p != a and wp[p] + 1 <= c), None)
        if a >= 0 and b is not None:
            O.debug_set_part(int(v), b)
            O.debug_set_part_weight(a, wp[a] - 1)
            O.debug_set_part_weight(b, wp[b] + 1)
            moved = True
            break
    assert moved
    assert O.check_invariants() is None
    assert _tag(O.check_invariants(O.cut() + 1)) == "I1"


def test_part_weights_equal_an_independent_recount():
    """ora_part_weights (maintained through apply / commits / rounds) equals
    a numpy recount from the exported labels and vertex weights, over a
    weighted stream with deletions, insertions and restoration."""
    g = gi.make_graph(4000, 64, 777, weighted=True)
    part = gi.block_partition(g.n, 5)
    O = oracle.Oracle(g.xadj, g.adjncy, 5, 0.03, part, g.vwgt, g.adjwgt)
    vw = list(g.vwgt)
    O.refine()
    S = gi.Stream(g, 5, weighted=True)
    for it in range(6):
        b = S.next(gi.MODE_MIX, 0.05)
        assert O.apply(b)[0] == 0
        vw += [int(m[3]) for m in b if m[0] == gi.VI]
        O.refine()
        p = O.partition()
        w = np.array(vw, np.int64)
        act = p >= 0
        rec = np.bincount(p[act], weights=w[act], minlength=5).astype(np.int64)
        assert np.array_equal(rec, O.part_weights()), it
        assert int(w[act].sum()) == O.total_weight()


# ---------------------------------------------------------------------------
# create-time validation: oracle and product (host-side, no GPU needed)
# ---------------------------------------------------------------------------
def _bad_inputs():
    ok_x = np.array([0, 1, 2, 2], np.int64)           # 0-1, vertex 2 isolated
    ok_a = np.array([1, 0], np.int32)
    p0 = np.zeros(3, np.int32)
    cases = {
        "self_loop": (np.array([0, 1, 1, 1], np.int64), np.array([0], np.int32), None, None, 2, 0.1, p0),
        "duplicate": (np.array([0, 2, 4, 4], np.int64), np.array([1, 1, 0, 0], np.int32), None, None, 2, 0.1, p0),
        "asymmetric": (np.array([0, 1, 1, 1], np.int64), np.array([1], np.int32), None, None, 2, 0.1, p0),
        "nbr_out_of_range": (np.array([0, 1, 2, 2], np.int64), np.array([5, 0], np.int32), None, None, 2, 0.1, p0),
        "nbr_negative": (np.array([0, 1, 2, 2], np.int64), np.array([-1, 0], np.int32), None, None, 2, 0.1, p0),
        "weight_asym": (ok_x, ok_a, None, np.array([1, 2], np.int32), 2, 0.1, p0),
        "edge_weight_zero": (ok_x, ok_a, None, np.array([0, 0], np.int32), 2, 0.1, p0),
        "edge_weight_256": (ok_x, ok_a, None, np.array([256, 256], np.int32), 2, 0.1, p0),
        "vertex_weight_zero": (ok_x, ok_a, np.array([1, 0, 1], np.int32), None, 2, 0.1, p0),
        "vertex_weight_65536": (ok_x, ok_a, np.array([1, 65536, 1], np.int32), None, 2, 0.1, p0),
        "part_ge_k": (ok_x, ok_a, None, None, 2, 0.1, np.array([0, 2, 0], np.int32)),
        "part_negative": (ok_x, ok_a, None, None, 2, 0.1, np.array([0, -1, 0], np.int32)),
        "k_1": (ok_x, ok_a, None, None, 1, 0.1, p0),
        "k_255": (ok_x, ok_a, None, None, 255, 0.1, p0),
        "eps_0": (ok_x, ok_a, None, None, 2, 0.0, p0),
        "eps_1.5": (ok_x, ok_a, None, None, 2, 1.5, p0),
        "eps_nan": (ok_x, ok_a, None, None, 2, float("nan"), p0),
        "xadj0_nonzero": (np.array([1, 2, 3, 3], np.int64), np.array([0, 1, 0], np.int32), None, None, 2, 0.1, p0),
        "xadj_decreasing": (np.array([0, 2, 1, 2], np.int64), np.array([1, 0], np.int32), None, None, 2, 0.1, p0),
    }
    return cases


@pytest.mark.parametrize("name", sorted(_bad_inputs()))
def test_oracle_create_rejects(name):
    xadj, adj, vw, aw, k, eps, part = _bad_inputs()[name]
    with pytest.raises(ValueError):
        oracle.Oracle(xadj, adj, k, eps, part, vw, aw)


def test_oracle_create_accepts_the_valid_baseline():
    ok_x = np.array([0, 1, 2, 2], np.int64)
    O = oracle.Oracle(ok_x, np.array([1, 0], np.int32), 2, 0.1, np.array([0, 1, 0], np.int32),
                      np.array([1, 65535, 1], np.int32), np.array([255, 255], np.int32))
    assert O.cut() == 255 and O.total_weight() == 65537


@pytest.mark.parametrize("name", sorted(_bad_inputs()))
def test_product_create_rejects_on_the_host(name):
    """igk_create validates the CSR on the host before any CUDA call, so the
    same table is checked on CPU: every input the oracle rejects is rejected
    by the product with IGK_EINVAL and no handle."""
    import paper_conf_dac_leejlczcshh25_b200 as igk
    xadj, adj, vw, aw, k, eps, part = _bad_inputs()[name]
    L = igk.lib()
    h = C.c_void_p()
    p = lambda a, t: None if a is None else a.ctypes.data_as(C.POINTER(t))  # noqa: E731
    s = L.igk_create(None, len(xadj) - 1, p(xadj, C.c_int64), p(adj, C.c_int32), p(vw, C.c_int32),
                     p(aw, C.c_int32), k, eps, p(part, C.c_int32), C.byref(h))
    assert s == igk.EINVAL and not h.value
