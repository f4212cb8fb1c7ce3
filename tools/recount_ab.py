#!/usr/bin/env python
"""Timing of k_recount (S9) on one graph.  The session-15 A/B of its variants
(env knobs since removed; results in profiles/r01_s15_recount_ab.txt) ran here.

Usage: recount_ab.py C2|C4 [iters]. The graph is built once; each variant is
timed over 15 launches with L2 flushed before each (median reported)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import igk_inputs as gi  # noqa: E402
import paper_conf_dac_leejlczcshh25_b200 as igk  # noqa: E402

cfgname = sys.argv[1] if len(sys.argv) > 1 else "C2"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 10
cfg = gi.CONFIGS[cfgname]
idx = int(cfgname[1:])
k = cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0]
g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(idx))
part, _ = gi.metis_partition(g, k)
G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part)
G.refine()
region0 = (part == 0).astype(np.int32) if cfg["mode"] == gi.MODE_ADVERSARIAL else None
S = gi.Stream(g, gi.stream_seed(gi.graph_seed(idx)), region0=region0)
for it in range(iters):
    G.apply(gi.next_batch(S, cfg))
    G.refine()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ss = G.store_stats()
b9 = ss["adj_entries"] * 5 + ss["n_total"] * 14
ref = None
VARIANTS = [("1", "0", "occ")]
for _rep in range(2):
    for pf, fast, bps in VARIANTS:
        os.environ["IGK_RECOUNT_MATCH"] = pf
        os.environ["IGK_RECOUNT_FAST"] = fast
        os.environ["IGK_RECOUNT_BPS"] = bps
        t = []
        for _ in range(15):
            flush.zero_()
            torch.cuda.synchronize()
            r = G.recount()
            t.append(G.last_ms()["recount"])
        if ref is None:
            ref = r
        assert r[0] == ref[0] and list(r[1]) == list(ref[1]), (pf, bps, r, ref)
        ms = float(np.median(t))
        print(f"{cfgname} match={pf} fast={fast} bps={bps} recount_ms={ms:.4f} GB/s={b9 / ms / 1e6:.0f} cut={r[0]}", flush=True)
