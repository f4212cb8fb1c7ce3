"""Side-by-side driver: CUDA path (through the C ABI) vs the CPU oracle on the
same seeded inputs; every comparison is bit-exact (integer-only method)."""
from __future__ import annotations

import numpy as np

import oracle
import paper_conf_dac_leejlczcshh25_b200 as igk

COMMON = ["affected", "inserted", "expanded", "filtered_in", "expanded_in", "evicted", "rounds",
          "moves_applied", "moves_deferred", "cut", "cap", "max_part_weight", "imbalanced"]


class Pair:
    """inv_every: run the oracle's invariant checker (I1-I5, with the GPU's
    maintained cut as the I1 operand) after every inv_every-th refine; the
    O(m log m) adjacency check I6 runs every struct_every-th refine."""

    def __init__(self, xadj, adjncy, k, eps, part, vwgt=None, adjwgt=None, check=True, inv_every=1,
                 struct_every=1, **kw):
        self.O = oracle.Oracle(xadj, adjncy, k, eps, part, vwgt, adjwgt)
        self.G = igk.IGKGraph(xadj, adjncy, k, eps, part, vwgt, adjwgt, check=check, **kw)
        self.k = k
        self.inv_every, self.struct_every = inv_every, struct_every
        self.n_refines = 0

    def invariants(self, gpu_cut, where=""):
        """north_star invariants after a refine, on the oracle's state, with
        the GPU's maintained cut checked against the oracle's recount (I1)."""
        self.n_refines += 1
        if not self.inv_every or self.n_refines % self.inv_every:
            return
        structure = bool(self.struct_every) and self.n_refines % self.struct_every == 0
        msg = self.O.check_invariants(gpu_cut, structure=structure)
        assert msg is None, f"{where}: invariant violated: {msg}"

    def compare_state(self, where="", full_csr=False):
        po, pg = self.O.partition(), self.G.partition()
        assert len(po) == len(pg), where
        if not np.array_equal(po, pg):
            bad = np.nonzero(po != pg)[0]
            raise AssertionError(f"{where}: {len(bad)} partition entries differ, first {bad[:8]} "
                                 f"oracle {po[bad[:8]]} gpu {pg[bad[:8]]}")
        assert self.O.cut() == self.G.cut(), where
        assert np.array_equal(self.O.part_weights(), self.G.part_weights()), where
        rc, rwp = self.G.recount()
        assert rc == self.G.cut(), f"{where}: maintained cut != recount"
        if full_csr:
            xo, ao, wo = self.O.export_csr()
            xg, ag, wg = self.G.export_csr()
            assert np.array_equal(xo, xg) and np.array_equal(ao, ag) and np.array_equal(wo, wg), where

    def apply(self, batch, where=""):
        so = self.O.apply(batch)
        sg = self.G.apply(batch)
        assert so[0] == sg[0], f"{where}: status oracle {so} gpu {sg}"
        assert so[1] == sg[1], where
        if so[0] != 0:
            assert so[2] == sg[2], f"{where}: bad index oracle {so[2]} gpu {sg[2]}"
        return so[0]

    def check_delta(self, pre, where=""):
        """igk_partition_delta == the oracle's label changes of the last
        refine: every vertex whose part now differs from its label before the
        refine (pending / inserted vertices included), deleted ones excluded."""
        post = self.O.partition()
        old = np.full(len(post), -2, np.int32)
        old[: len(pre)] = pre
        idx = np.nonzero((post >= 0) & (post != old))[0]
        d = self.G.partition_delta()
        got = d[np.argsort(d[:, 0], kind="stable")] if len(d) else d.reshape(0, 2)
        exp = np.stack([idx, post[idx]], axis=1).astype(np.int32)
        assert got.shape == exp.shape and np.array_equal(got, exp), \
            f"{where}: delta differs ({len(got)} gpu pairs vs {len(exp)} expected)"

    def refine(self, where=""):
        pre = self.O.partition()
        so, sto = self.O.refine()
        sg, stg = self.G.refine()
        assert so == sg, where
        diff = {f: (sto[f], stg[f]) for f in COMMON if sto[f] != stg[f]}
        assert not diff, f"{where}: stats differ (oracle, gpu): {diff}"
        self.invariants(stg["cut"], where)
        self.check_delta(pre, where)
        return sto, stg

    def refine_global(self, where=""):
        pre = self.O.partition()
        so, sto = self.O.refine_global()
        sg, stg = self.G.refine_global()
        assert so == sg, where
        diff = {f: (sto[f], stg[f]) for f in COMMON if sto[f] != stg[f]}
        assert not diff, f"{where}: global refine stats differ (oracle, gpu): {diff}"
        self.invariants(stg["cut"], where)
        self.check_delta(pre, where)
        return sto, stg


    def repartition(self, where=""):
        """NEXT-2 F8 on both sides: partitions, cut and W_p equal afterwards."""
        assert self.O.repartition() == 0, where
        cut = self.G.repartition()
        assert cut == self.O.cut(), f"{where}: repartition cut gpu {cut} oracle {self.O.cut()}"
        msg = self.O.check_invariants(cut)
        assert msg is None, f"{where}: invariant violated after repartition: {msg}"
        self.compare_state(where)
        return cut


def run_stream(pair: Pair, batches, full_csr_every=0, tag=""):
    stats = []
    for it, b in enumerate(batches):
        st = pair.apply(b, f"{tag} it{it} apply")
        assert st == 0
        pair.compare_state(f"{tag} it{it} after apply",
                           full_csr=bool(full_csr_every) and it % full_csr_every == 0)
        sto, stg = pair.refine(f"{tag} it{it} refine")
        pair.compare_state(f"{tag} it{it} after refine")
        stats.append(stg)
    return stats
