"""Time the GPU full partitioner (igk_fgp_partition) on the BASELINE graphs
and compare its cut with METIS (DESIGN.md 4 F6 / 7).  Prints one JSON line per
configuration."""
import json
import sys
import time

import numpy as np

import igk_inputs as gi
import paper_conf_dac_leejlczcshh25_b200 as igk

CFGS = {"c1": (10000, 4, 64), "c2": (1000000, 4, 1024), "c4": (10000000, 16, 4096)}


def cut_of(g, part):
    src = np.repeat(np.arange(g.n), np.diff(g.xadj))
    return int((part[src] != part[g.adjncy]).sum()) // 2


for name in (sys.argv[1:] or ["c1", "c2"]):
    n, k, fmax = CFGS[name]
    g = gi.make_graph(n, fmax, gi.graph_seed({"c1": 0, "c2": 1, "c4": 3}[name]))
    igk.fgp_partition(g.xadj, g.adjncy, k, 0.03)  # warm-up
    ts = []
    for _ in range(3):
        t0 = time.perf_counter()
        part, lv = igk.fgp_partition(g.xadj, g.adjncy, k, 0.03)
        ts.append(time.perf_counter() - t0)
    t0 = time.perf_counter()
    _, mcut = gi.metis_partition(g, k)
    tm = time.perf_counter() - t0
    pw = np.bincount(part, minlength=k)
    print(json.dumps({"config": name, "n": n, "k": k, "fgp_ms": round(1e3 * min(ts), 2), "levels": lv,
                      "fgp_cut": cut_of(g, part), "metis_cut": mcut, "metis_ms_host": round(1e3 * tm, 1),
                      "max_part_w": int(pw.max()), "W": n}), flush=True)
