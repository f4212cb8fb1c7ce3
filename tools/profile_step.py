#!/usr/bin/env python
"""Short run of the fused step (igk_step = k_step) for ncu captures:
create, settle, then `iters` iterations of config `cfg` (bench's workload,
rank 0).  Usage: python tools/profile_step.py C4 4 [k] [frac]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import igk_inputs as gi  # noqa: E402
import paper_conf_dac_leejlczcshh25_b200 as igk  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 4
cfg = dict(gi.CONFIGS[name])
k = int(sys.argv[3]) if len(sys.argv) > 3 else (cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0])
if len(sys.argv) > 4:
    cfg["frac"] = float(sys.argv[4])
elif isinstance(cfg.get("frac"), tuple):
    cfg["frac"] = cfg["frac"][2]
idx = int(name[1:])
g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(idx))
part, _ = gi.metis_partition(g, k)
G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part)
G.refine()
region0 = (part == 0).astype(np.int32) if cfg["mode"] == gi.MODE_ADVERSARIAL else None
S = gi.Stream(g, gi.stream_seed(gi.graph_seed(idx)), region0=region0)
for it in range(iters):
    _, st, _ = G.step(gi.next_batch(S, cfg))
    print(it, "affected", st["affected"], "rounds", st["rounds"], "ms", G.last_ms())
print("done", G.cut())
rc = G.recount()  # S9 full-store scan (k_recount), captured by `ncu -k regex:k_recount`
assert rc[0] == G.cut(), (rc, G.cut())
print("recount ok", rc[0])
