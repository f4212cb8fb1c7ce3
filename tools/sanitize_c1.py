#!/usr/bin/env python
"""A short C1 run through every single-GPU entry point, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck): create, settle, apply +
refine, fused step, pipelined step, global refine, recount (both S9 kernels),
delta, export, compaction.  Checks the results against the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import igk_inputs as gi  # noqa: E402
from tests.parity import Pair  # noqa: E402

cfg = gi.CONFIGS["C1"]
g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(1))
part, _ = gi.metis_partition(g, 4)
P = Pair(g.xadj, g.adjncy, 4, cfg["eps"], part, check=True)
P.refine("settle")
S = gi.Stream(g, gi.stream_seed(gi.graph_seed(1)))
for it in range(4):
    b = gi.next_batch(S, cfg)
    if it == 0:
        assert P.apply(b) == 0
        P.refine("it0")
    elif it == 1:
        P.O.apply(b)
        P.O.refine()
        assert P.G.step(b)[0] == 0
    elif it == 2:
        P.O.apply(b)
        P.O.refine()
        P.G.stage_batch(b)
        P.G.step_begin()
        assert P.G.step_end()[0] == 0
    else:
        assert P.apply(b) == 0
        P.refine_global("global")
    P.compare_state(f"it{it}", full_csr=(it == 3))
    P.G.partition_delta()
from paper_conf_dac_leejlczcshh25_b200 import IGKGraph  # noqa: E402
for variant in ("tma", "gather"):  # the A/B S9 kernels (the default k_recount3 ran in check mode above)
    os.environ["IGK_RECOUNT"] = variant
    G2 = IGKGraph(g.xadj, g.adjncy, 4, cfg["eps"], part)
    assert G2.recount()[0] == G2.cut()
    G2.close()
os.environ.pop("IGK_RECOUNT")
# weighted handle: k_recount3<true> (edge weights 2, vertex weights 3)
G3 = IGKGraph(g.xadj, g.adjncy, 4, cfg["eps"], part, vwgt=np.full(g.n, 3, np.int32),
              adjwgt=np.full(len(g.adjncy), 2, np.int32))
c3, w3 = G3.recount()
assert c3 == G3.cut() and c3 == 2 * G2.cut(), (c3, G3.cut())
G3.close()
P.G.compact()
P.compare_state("compacted", full_csr=True)
print("sanitize run ok, cut", P.G.cut())
