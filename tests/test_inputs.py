"""Generator sanity + medium-scale oracle invariants (CPU only)."""
import numpy as np

import igk_inputs as gi
import oracle


def test_graph_shape_c1():
    g = gi.make_graph(10_000, 64, gi.graph_seed(1))
    deg = np.diff(g.xadj)
    assert 3.0 <= deg.mean() <= 5.0          # circuit-like average degree
    assert deg.max() >= 8 * deg.mean()       # heavy-tailed fanout
    # symmetric + simple: the oracle's create() validates both
    oracle.Oracle(g.xadj, g.adjncy, 4, 0.03, gi.block_partition(g.n, 4))


def test_generator_is_deterministic():
    a = gi.make_graph(5000, 64, 7)
    b = gi.make_graph(5000, 64, 7)
    assert np.array_equal(a.xadj, b.xadj) and np.array_equal(a.adjncy, b.adjncy)
    sa, sb = gi.Stream(a, 11), gi.Stream(b, 11)
    for _ in range(3):
        assert np.array_equal(sa.next(gi.MODE_MIX, 0.01), sb.next(gi.MODE_MIX, 0.01))


def test_c1_stream_valid_and_invariants():
    cfg = gi.CONFIGS["C1"]
    g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(1))
    part, _ = gi.metis_partition(g, cfg["k"])
    O = oracle.Oracle(g.xadj, g.adjncy, cfg["k"], cfg["eps"], part)
    O.refine()
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(1)))
    for it in range(cfg["iters"]):
        b = gi.next_batch(S, cfg)
        kinds = np.bincount(b[:, 0], minlength=4)
        assert kinds[1] == 100 and kinds[2] == 100 and kinds[0] == 200 and kinds[3] == 200
        st, fid, bad = O.apply(b)
        assert st == 0, bad
        s, stats = O.refine()
        assert s == 0
        assert O.check_invariants() is None
        assert stats["max_part_weight"] <= stats["cap"]
        assert O.n_total == S.n_total


def test_weighted_and_adversarial_streams_valid():
    g = gi.make_graph(4000, 64, 3, weighted=True)
    part = gi.block_partition(g.n, 8)
    O = oracle.Oracle(g.xadj, g.adjncy, 8, 0.03, part, g.vwgt, g.adjwgt)
    O.refine()
    S = gi.Stream(g, 5, weighted=True, region0=(part == 0).astype(np.int32))
    evicted = 0
    for it in range(8):
        b = S.next(gi.MODE_ADVERSARIAL, 0.0, 40, 20, 0, 0)
        st, fid, bad = O.apply(b)
        assert st == 0, bad
        s, stats = O.refine()
        evicted += stats["evicted"]
        assert O.check_invariants() is None
    assert evicted > 0


def test_adversarial_batch_needs_region0():
    """MODE_ADVERSARIAL draws deletions from part 0; without the region the
    generator has nothing to draw from, so next_batch refuses (no crash)."""
    import pytest
    g = gi.make_graph(2000, 64, 5)
    S = gi.Stream(g, 3)
    with pytest.raises(ValueError):
        gi.next_batch(S, dict(gi.CONFIGS["C5"], literal=dict(nvd=10, nvi=10)))
