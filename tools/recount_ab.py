#!/usr/bin/env python
"""A/B of the S9 cut / W_p reduction kernels on one store: k_recount3 (the
default, "v3"), the round-1 direct-gather k_recount (IGK_RECOUNT=gather) and
the TMA-pipelined k_recount_tma (IGK_RECOUNT=tma); the variant is read at
igk_create.  Prints median kernel ms (L2 flushed before each launch) and the
algorithmic-bytes bandwidth of bench.py's S9 line.
Usage: python tools/recount_ab.py C4 [reps] [variants, comma-separated]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import igk_inputs as gi  # noqa: E402
import paper_conf_dac_leejlczcshh25_b200 as igk  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 9
cfg = dict(gi.CONFIGS[name])
k = cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0]
idx = int(name[1:])
g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(idx))
part, _ = gi.metis_partition(g, k)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
out = {}
variants = sys.argv[3].split(",") if len(sys.argv) > 3 else ["v3", "gather", "tma"]
for variant in variants:
    os.environ["IGK_RECOUNT"] = variant
    G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part)
    G.refine()
    ts, cut = [], None
    for _ in range(reps):
        flush.zero_()
        torch.cuda.synchronize()
        c, _ = G.recount()
        ts.append(G.last_ms()["recount"])
        assert cut is None or c == cut
        cut = c
    ss = G.store_stats()
    by = ss["adj_entries"] * 4 + ss["adj_entries"] // 2 + ss["n_active"] * 17
    ms = float(np.median(ts))
    out[variant] = {"ms": ms, "cut": cut, "bytes": by, "gbs": by / ms / 1e6, "frac": by / ms / 1e6 / peak}
    print(name, variant, json.dumps(out[variant]), flush=True)
    G.close()
assert len({o["cut"] for o in out.values()}) == 1, out
if "v3" in out and "gather" in out:
    print(name, "speedup v3 vs gather", out["gather"]["ms"] / out["v3"]["ms"])
