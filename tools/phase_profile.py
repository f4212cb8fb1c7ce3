#!/usr/bin/env python
"""Average per-phase durations inside k_apply / k_refine (globaltimer stamps)
over C2 iterations.  Usage: python tools/phase_profile.py [iters] [config] [k] [frac]
(IGK_FLUSH=1: L2 flushed before every iteration; IGK_DEBUG_ARRIVALS=1: per-CTA barrier arrivals)"""
import os
import sys
from collections import defaultdict

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ.setdefault("IGK_DEBUG_PHASES", "1")
sys.path.insert(0, ROOT)
import igk_inputs as gi  # noqa: E402
import paper_conf_dac_leejlczcshh25_b200 as igk  # noqa: E402

NAMES = {100: "start", 101: "V1 hash/counts", 102: "V2 validate/alloc", 103: "M12 deletions",
         104: "M3 compact/insert-vertices", 199: "M4 insert-edges",
         200: "start", 201: "F0 R1 filter", 202: "F1 commit C1 + expand", 203: "F2 R2 filter",
         204: "F3 commit C2"}


def main():
    iters = int(sys.argv[1]) if len(sys.argv) > 1 else 30
    name = sys.argv[2] if len(sys.argv) > 2 else "C2"
    cfg = dict(gi.CONFIGS[name])
    k = int(sys.argv[3]) if len(sys.argv) > 3 else (cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0])
    if len(sys.argv) > 4:
        cfg["frac"] = float(sys.argv[4])
    idx = int(name[1:])
    g = gi.make_graph(cfg["n"], cfg["fmax"], gi.graph_seed(idx))
    part, _ = gi.metis_partition(g, k)
    G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part)
    G.refine()
    region0 = (part == 0).astype(np.int32) if cfg["mode"] == gi.MODE_ADVERSARIAL else None
    S = gi.Stream(g, gi.stream_seed(gi.graph_seed(idx)), region0=region0)
    acc = [defaultdict(list), defaultdict(list)]
    tot = [[], []]
    flush = None
    if os.environ.get("IGK_FLUSH"):  # L2 flushed before every iteration, as in bench.py
        import torch
        flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for it in range(iters):
        if flush is not None:
            flush.zero_()
            torch.cuda.synchronize()
        G.apply(gi.next_batch(S, cfg, cfg.get("frac") if cfg["mode"] == gi.MODE_MIX else None))
        pa = G.phase_times(0)
        _, st = G.refine()
        pr = G.phase_times(1)
        if os.environ.get("IGK_DEBUG_ARRIVALS") and it >= iters - 3:
            print(f"k_refine arrivals, iteration {it}:")
            arrivals_report(G, 1)
        if it < 3:
            continue
        for w, ph in enumerate((pa, pr)):
            for (i0, t0), (i1, t1) in zip(ph, ph[1:]):
                acc[w][(i1, NAMES.get(i1, f"phase {i1}"))].append((t1 - t0) / 1e3)
            tot[w].append((ph[-1][1] - ph[0][1]) / 1e3)
    ms = G.last_ms()
    for w, name in enumerate(("k_apply", "k_refine")):
        print(f"{name}: stamped span {np.mean(tot[w]):.1f} us (event-timed last launch {ms['apply' if w == 0 else 'refine'] * 1e3:.1f} us)")
        for key, v in sorted(acc[w].items(), key=lambda kv: kv[0][0]):
            print(f"   {key[0]:4d} {key[1]:32s} n={len(v):4d} mean {np.mean(v):7.2f} us")




def arrivals_report(G, which):
    """Per barrier slot: spread of CTA arrivals and the slowest CTA."""
    A = G.arrivals(which)
    if A is None:
        return
    ph = dict(G.phase_times(which))
    t0 = min(v for v in A.flatten() if v > 0)
    slow = {}
    for s in range(128):
        row = A[s]
        if not row.any():
            continue
        r = (row - t0) / 1e3
        slow[s] = int(np.argmax(row))
        print(f"   slot {s:3d}: arrivals min {r.min():8.2f} med {np.median(r):8.2f} max {r.max():8.2f} us, "
              f"slowest CTA {slow[s]}")
    W = G.arrivals(2)  # per warp: F1 commit-pass end time, heaviest prefix
    if W is not None and W[0].any():
        t = (W[0] - t0) / 1e3
        order = np.argsort(-t)[:5]
        tin = np.where(W[2] > 0, (W[2] - t0) / 1e3, np.nan)
        tout = np.where(W[3] > 0, (W[3] - t0) / 1e3, np.nan)
        print("   F1 commit pass, latest warps (cta.warp: end us, heaviest prefix, warp-path commit, mark item,"
              " lane-0 item enter/exit us):",
              "; ".join(f"{i // 16}.{i % 16}: {t[i]:.2f}, {W[1][i] & 0xfffff}, {bool(W[1][i] >> 20 & 1)}, "
                        f"{bool(W[1][i] >> 21 & 1)}, {tin[i]:.2f}/{tout[i]:.2f}" for i in order))
        ok = ~np.isnan(tin)
        if ok.any():
            print(f"   lane-0 thread items: enter median {np.nanmedian(tin):.2f} p90 {np.nanpercentile(tin, 90):.2f}; "
                  f"body median {np.nanmedian(tout - tin):.2f} p90 {np.nanpercentile(tout - tin, 90):.2f} max "
                  f"{np.nanmax(tout - tin):.2f} us")
        print(f"   F1 commit pass warp ends: median {np.median(t):.2f} us, p90 {np.percentile(t, 90):.2f} us")
    # sub-phase stamps (slots 110-114) of the CTAs that closed F0 (slot 1) and F1 (slot 2) last
    for bar, subs in ((1, (113, 114)), (2, (110, 111, 112))):
        if bar in slow and all(x in slow for x in subs):
            c = slow[bar]
            print(f"   slowest CTA {c} at barrier slot {bar}: " +
                  ", ".join(f"slot {x} at {(A[x][c] - t0) / 1e3:.2f} us" for x in subs))


if __name__ == "__main__":
    main()
