#!/usr/bin/env python
"""Long-stream endurance run (store maintenance).

Drives one graph through many incremental iterations of a BASELINE config with
the fused step (host batches), printing the store occupancy and the per-step
device time every `--every` iterations; checks the maintained cut against a
full recount at those points.  Vertex IDs are never reused and relocations
leave holes in the slab, so a stream this long must go through the automatic
capacity growth / compaction path.

  python tools/long_run.py [--config C2] [--iters 3000] [--every 250]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import igk_inputs as gi  # noqa: E402
import paper_conf_dac_leejlczcshh25_b200 as igk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--iters", type=int, default=3000)
    ap.add_argument("--every", type=int, default=250)
    a = ap.parse_args()
    cfg = dict(gi.CONFIGS[a.config])
    idx = int(a.config[1:])  # graph_seed index as in tests / bench
    k = cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0]
    g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(idx))
    part, _ = gi.metis_partition(g, k)
    G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part, g.vwgt, g.adjwgt)
    G.refine()
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(idx)))
    ms, t0 = [], time.time()
    for it in range(a.iters):
        b = gi.next_batch(S, cfg)
        st, stats, bad = G.step(b)
        assert st in (0, 6) and bad == -1, (it, st, bad)
        ms.append(G.last_ms()["refine"])  # fused step: whole step timed as one kernel
        if (it + 1) % a.every == 0 or it + 1 == a.iters:
            rc, _ = G.recount()
            assert rc == G.cut(), (it, rc, G.cut())
            w = ms[-a.every:]
            print(json.dumps({"it": it + 1, "cut": G.cut(), **G.store_stats(),
                              "ms_step_med": sorted(w)[len(w) // 2], "ms_step_max": max(w),
                              "wall_s": round(time.time() - t0, 1)}), flush=True)


if __name__ == "__main__":
    main()
