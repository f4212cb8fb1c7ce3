#!/usr/bin/env python
"""Short C2 run for ncu captures: create, settle, then `iters` iterations."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import igk_inputs as gi  # noqa: E402
import paper_conf_dac_leejlczcshh25_b200 as igk  # noqa: E402

cfgname = sys.argv[1] if len(sys.argv) > 1 else "C2"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 4
cfg = gi.CONFIGS[cfgname]
idx = int(cfgname[1:])
k = cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0]
g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(idx))
part, _ = gi.metis_partition(g, k)
G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part)
G.refine()
S = gi.Stream(g, gi.stream_seed(gi.graph_seed(idx)))
for it in range(iters):
    G.apply(gi.next_batch(S, cfg))
    G.refine()
if "--recount" in sys.argv:
    import torch
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        flush.zero_()
        torch.cuda.synchronize()
        G.recount()
    print("recount ms", G.last_ms()["recount"], G.store_stats())
print("done", G.cut())
