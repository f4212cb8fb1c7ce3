#!/usr/bin/env python
"""bench.py -- iG-kway incremental refinement on B200 (BASELINE.json metric).

One step = one incremental iteration = igk_apply_modifiers + igk_refine over one
seeded synthetic modifier batch (all SURVEY 8(a) rows: S1 apply/mark, S2-S4
filter/expansion, S5 restoration when a part is overweight, S6-S8 rounds).
Default workload = BASELINE configs[1] (C2): 1M-vertex circuit-shaped graph,
k=4, eps=3%, 1% modified vertices per iteration.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl reference]

value       = affected vertices/s (whole job), device-resident batches, CUDA events
ms_per_step = device ms per incremental iteration (apply + refine)
e2e         = same metric through the public C ABI with HOST batches (H2D of the
              batch + D2H of the cut inside the timed region)
--impl reference = the CPU oracle (oracle/) timed on this host (the slow arm).
Multi-GPU: by default ONE C4 graph vertex-range sharded
over the N ranks (igk_options.nranks/rank/nccl_id: the library's own NCCL
communicator; fixed-size all-reduces of candidate bitmaps and per-round move
records), strong scaling, device time max over ranks; --replicas runs N
independent instances (weak scaling).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import benchdist  # noqa: E402
import igk_inputs as gi  # noqa: E402

METRIC = "ms per incremental iteration & affected vertices/s; cut vs full repartition"
UNIT = "affected vertices/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=None,
                    help="workload (default: C2 at N=1; C4 vertex-range sharded at N>1)")
    ap.add_argument("--k", type=int, default=0)
    ap.add_argument("--frac", type=float, default=0.0)
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--cpu-iters", type=int, default=150, help="oracle sample size (iterations)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--no-repartition", action="store_true", help="skip the METIS full-repartition comparison")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no e2e/cpu legs)")
    ap.add_argument("--shard", action="store_true",
                    help="ONE graph vertex-range sharded over the ranks (the default at N>1; strong scaling; "
                         "at N=1 the sharded protocol runs on one rank over an NCCL loopback communicator)")
    ap.add_argument("--p2p", action="store_true",
                    help="sharded: all rounds of a refine in one persistent kernel per rank, move records "
                         "stored into peer memory + device barrier (NEXT-3) instead of per-round all-reduces")
    ap.add_argument("--replicas", action="store_true",
                    help="N>1: independent graph instances per rank (weak scaling) instead of sharding")
    return ap.parse_args()


def workload(args, rank):
    if args.shard:
        rank = 0  # every rank holds the same (canonical) graph
    idx = int(args.config[1:])
    cfg = dict(gi.CONFIGS[args.config])
    n = args.n or cfg["n"]
    k = args.k or (cfg["k"] if isinstance(cfg["k"], int) else cfg["k"][0])
    frac = args.frac or (cfg.get("frac") if not isinstance(cfg.get("frac"), tuple) else cfg["frac"][2])
    gseed = benchdist.rank_graph_seed(idx, rank)  # rank 0 = the canonical instance
    g = gi.make_graph(n, cfg["fmax"], gseed)
    part, metis_cut = gi.metis_partition(g, k)
    region0 = (part == 0).astype(np.int32) if cfg["mode"] == gi.MODE_ADVERSARIAL else None
    S = gi.Stream(g, gi.stream_seed(gseed), region0=region0)
    cfg = dict(cfg, frac=frac)
    desc = (f"{args.config}: {n}-vertex circuit-shaped graph (avg deg ~4, fanout <= {cfg['fmax']}), "
            f"k={k}, eps={cfg['eps']}, " +
            (f"{frac * 100:g}% modified vertices per iteration" if cfg["mode"] == gi.MODE_MIX else "literal batch mix"))
    return g, part, metis_cut, S, cfg, k, desc


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.samples = []
        self._stop = False

    def start(self):
        def run():
            while not self._stop:
                try:
                    out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                         timeout=5).stdout.strip()
                    if out:
                        self.samples.append([x.strip() for x in out.split(",")])
                except Exception:
                    pass
                time.sleep(0.1)
        self.t = threading.Thread(target=run, daemon=True)
        self.t.start()

    def stop(self):
        self._stop = True
        self.t.join(timeout=10)
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[3 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"], "measured"
    except Exception:
        return 6650.0, "fallback"


def refine_bytes(st, weighted=False):
    """Algorithmic bytes of one k_refine launch: every scanned
    adjacency entry = 4 B neighbour ID + 1 B label gather (+4 B weight), every
    touched vertex = 16 B of per-vertex state (offset, degree, label, flags,
    list entry)."""
    per_entry = 5 + (4 if weighted else 0)
    touched = st["affected"] + st["expanded"] + st["moves_applied"] + st["moves_deferred"] + st["evicted"]
    return st["adj_entries_scanned"] * per_entry + touched * 16


def host_cpu():
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return model, os.cpu_count()


class pinned_to_one_core:
    """taskset-equivalent: run the block on ONE host core (the oracle is
    single-threaded by construction; pinning makes 'cores: 1' literal)."""

    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        self.core = max(self.old)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *a):
        os.sched_setaffinity(0, self.old)


def cpu_baseline(g, part, k, eps, batches, gpu_cuts, iters):
    import oracle
    n_it = min(iters, len(batches))
    model, ncpu = host_cpu()
    pin = pinned_to_one_core().__enter__()
    t0 = time.perf_counter()
    O = oracle.Oracle(g.xadj, g.adjncy, k, eps, part)
    O.refine()
    t_setup = time.perf_counter() - t0
    aff, tt, cut_ok = 0, 0.0, True
    for i in range(n_it):
        t = time.perf_counter()
        O.apply(batches[i])
        _, st = O.refine()
        tt += time.perf_counter() - t
        aff += st["affected"]
        if i < len(gpu_cuts) and gpu_cuts[i] != st["cut"]:
            cut_ok = False
    pin.__exit__()
    return {"value": aff / tt, "unit": UNIT, "cores": 1, "kind": "oracle",
            "host_cpu": model, "host_nproc": ncpu, "taskset_core": pin.core,
            "sample": f"first {n_it} iterations of the same workload (apply+refine, single-threaded, "
                      f"pinned to core {pin.core} of {ncpu}; {tt:.1f}s; setup {t_setup:.1f}s excluded)",
            "ms_per_iteration": 1e3 * tt / n_it,
            "parity_cut_checked_iters": min(n_it, len(gpu_cuts)), "parity_cut_match": cut_ok}


PH_NAMES = {220: "boundary", 201: "F0_filter", 202: "F1_commit_expand", 203: "F2_filter", 204: "F3_commit",
            205: "R3_restore", 206: "R3_restore", 207: "R3_restore", 208: "round_gain", 209: "round_move",
            210: "round_move", 212: "round_move", 213: "round_move", 211: "epilogue"}


def phase_profile(G, batches_dev, peak):
    """Per-phase roofline of the refine (verdict r1 item 3):
    profile mode records a %globaltimer stamp after every grid barrier and,
    per phase, the adjacency entries scanned and list items processed.
    Algorithmic bytes of a phase = 5 B per scanned entry (4 B neighbour ID +
    1 B label gather) + 16 B per list item (its vertex record / list entry);
    time = the phase's stamp interval (barrier included).  Run AFTER the timed
    region on further iterations of the same stream (profile mode replaces
    the step's completion notice by a full control-block copy)."""
    G.set_profile(True)
    acc = {}
    for ptr, cnt in batches_dev:
        G.step_device(ptr, cnt)
        st = G.phase_times(1)
        work = G.phase_work()
        prev = st[0][1] if st else 0
        for pid, t in st[1:]:
            name = PH_NAMES.get(pid)  # sub-phase stamps (select passes) merge into the next named one
            if name:
                a = acc.setdefault(name, {"ns": 0, "scanned": 0, "items": 0})
                a["ns"] += t - prev
                prev = t
        for name, (sc, it) in work.items():
            a = acc.setdefault(name, {"ns": 0, "scanned": 0, "items": 0})
            a["scanned"] += sc
            a["items"] += it
    G.set_profile(False)
    n = max(len(batches_dev), 1)
    out = {}
    for name, a in acc.items():
        if a["ns"] == 0 and a["scanned"] == 0:
            continue
        by = 5 * a["scanned"] + 16 * a["items"]
        us = a["ns"] / 1e3 / n
        gbs = by / n / (a["ns"] / n) if a["ns"] else 0.0  # bytes per ns = GB/s
        out[name] = {"us": round(us, 2), "bytes": int(by / n), "gbs": round(gbs, 2), "frac": gbs / peak}
    gm = [out[x] for x in ("round_gain", "round_move") if x in out]
    gain_move = None
    if gm:
        by = sum(x["bytes"] for x in gm)
        us = sum(x["us"] for x in gm)
        gain_move = {"bytes": by, "us": round(us, 2), "gbs": by / (us * 1e3) if us else 0.0,
                     "frac": (by / (us * 1e3)) / peak if us else 0.0}
    return {"iterations": n, "phases": out, "gain_move": gain_move,
            "bytes_rule": "5 B per scanned adjacency entry + 16 B per list item; time = stamp interval"}


def full_repartition(G, k, igk_cut, ms_per_step):
    """The metric's "cut vs full repartition": METIS k-way
    (default options, ufactor 30 = the same 3% imbalance) from scratch on the
    CURRENT graph (exported from the device store, deleted IDs dropped and the
    active vertices relabelled densely), single-threaded on the host.  Reports
    both cuts and the repartition wall time against one incremental step."""
    xadj, adj, w = G.export_csr(sort_rows=False)
    part = G.partition()
    act = part >= 0
    new_id = np.cumsum(act) - 1
    deg = np.diff(xadj)[act]
    cx = np.zeros(int(act.sum()) + 1, dtype=np.int64)
    np.cumsum(deg, out=cx[1:])
    # inactive rows are empty (I6), so the exported entries are exactly the active rows' entries
    assert int(xadj[-1]) == int(deg.sum()), "exported CSR has entries in deleted rows"
    ca = new_id[adj].astype(np.int32)
    g = gi.Graph(cx, ca, None, None if (w == 1).all() else w.astype(np.int32))
    t = time.perf_counter()
    mpart, mcut = gi.metis_partition(g, k)
    t_metis = time.perf_counter() - t
    # NEXT-1: one global boundary refinement (igk_refine_global) on the
    # same graph -- how much of the incremental drift it recovers, and at what cost
    import torch
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    _, gst = G.refine_global()
    e1.record()
    torch.cuda.synchronize()
    gcut = G.cut()
    # NEXT-2: the GPU full partitioner (IGK-FGP v1) on the same graph, in
    # place (igk_repartition: device export + coarsening + LP uncoarsening)
    t = time.perf_counter()
    fcut = G.repartition()
    torch.cuda.synchronize()
    t_fgp = time.perf_counter() - t
    return {"igk_cut": int(igk_cut), "metis_cut": int(mcut), "cut_ratio": igk_cut / max(mcut, 1),
            "metis_s": t_metis, "metis_vs_step": 1e3 * t_metis / ms_per_step,
            "global_refine": {"cut": int(gcut), "cut_ratio": gcut / max(mcut, 1), "ms": e0.elapsed_time(e1),
                              "boundary_affected": gst["affected"], "rounds": gst["rounds"]},
            "gpu_fgp": {"cut": int(fcut), "cut_ratio": fcut / max(mcut, 1), "ms": 1e3 * t_fgp,
                        "vs_step": 1e3 * t_fgp / ms_per_step, "how": "igk_repartition (group size 6), wall clock"},
            "n_active": int(act.sum()), "how": "METIS_PartGraphKway default options (ufactor 30), 1 host core, "
                                               "on the graph as it stands after the timed iterations"}


def run_reference(args, rank, world):
    if rank != 0:
        return
    g, part, metis_cut, S, cfg, k, desc = workload(args, 0)
    import oracle
    batches = [gi.next_batch(S, cfg) for _ in range(args.warmup + args.steps)]
    O = oracle.Oracle(g.xadj, g.adjncy, k, cfg["eps"], part)
    O.refine()
    for i in range(args.warmup):
        O.apply(batches[i])
        O.refine()
    aff, tt = 0, 0.0
    model, ncpu = host_cpu()
    with pinned_to_one_core() as pin:
        for i in range(args.warmup, args.warmup + args.steps):
            t = time.perf_counter()
            O.apply(batches[i])
            _, st = O.refine()
            tt += time.perf_counter() - t
            aff += st["affected"]
    v = aff / tt
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tt / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic", "config": {"workload": desc, "n": g.n, "k": k},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "host_cpu": model,
                             "host_nproc": ncpu, "taskset_core": pin.core,
                             "sample": f"{args.steps} timed iterations after {args.warmup} warm-up, "
                                       f"pinned to core {pin.core} of {ncpu}"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    rank, world, local = benchdist.env_ranks()
    if world > 1 and not args.replicas:
        args.shard = True
    if args.config is None:
        args.config = "C4" if (args.shard and world > 1) else "C2"
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import torch
    import paper_conf_dac_leejlczcshh25_b200 as igk
    one_gpu_test = os.environ.get("IGK_BENCH_ONE_GPU") == "1"  # plumbing test: all ranks on cuda:0 over gloo
    if one_gpu_test:
        local = 0
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if one_gpu_test:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    g, part, metis_cut, S, cfg, k, desc = workload(args, rank)
    W, K = args.warmup, args.steps
    e2e_steps = 0 if args.profile else K
    n_prof = 0 if (args.profile or args.shard) else 5
    batches = [gi.next_batch(S, cfg) for _ in range(W + K + e2e_steps + (1 if e2e_steps else 0) + n_prof)]
    stream = torch.cuda.current_stream()
    shard_kw = {}
    if args.shard:  # every rank: the same graph, its own vertex range; the library's NCCL communicator
        if one_gpu_test:
            shard_kw = dict(nranks=world, rank=rank, comm=igk.TorchComm())
        else:
            uid = [igk.nccl_unique_id() if rank == 0 else None]
            if dist:
                dist.broadcast_object_list(uid, src=0)
            shard_kw = dict(nranks=world, rank=rank, nccl_id=uid[0])
        shard_kw["p2p"] = args.p2p
    G = igk.IGKGraph(g.xadj, g.adjncy, k, cfg["eps"], part, device=local, stream=stream.cuda_stream, **shard_kw)
    G.refine()  # settle the METIS partition (untimed; collective when sharded)
    dev_batches = [torch.from_numpy(b).cuda() for b in batches[: W + K]]
    flush = None if args.no_flush else torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    gpu_cuts = []
    st_buf = igk.Stats()
    def one_step(i, b):  # igk_step_device: apply + refine (collective on a sharded handle)
        G.step_device(dev_batches[i].data_ptr(), len(b), st_buf)
        return {f: int(getattr(st_buf, f)) for f in igk.STATS}

    deg_start = round(2.0 * g.m / g.n, 3)
    for i in range(W):
        gpu_cuts.append(one_step(i, batches[i])["cut"])
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    l0 = G.kernel_launches()
    clk = ClockSampler(local)
    clk.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    aff, refine_ms, apply_ms, rbytes, stats = 0, 0.0, 0.0, 0, []
    for i in range(K):
        b = batches[W + i]
        if flush is not None:
            flush.zero_()  # L2 flush (256 MiB > 126 MB L2), outside the timed events
        ev[i][0].record(stream)
        st = one_step(W + i, b)
        ev[i][1].record(stream)
        ms = G.last_ms()
        refine_ms += ms["refine"] + ms["apply"]  # igk_step: ONE fused k_step (apply_ms 0); sharded: both halves
        apply_ms += ms["apply"]
        aff += st["affected"]
        rbytes += refine_bytes(st) + 16 * len(b)  # + the batch itself
        stats.append(st)
        gpu_cuts.append(st["cut"])
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    clocks = clk.stop()
    launches = G.kernel_launches() - l0
    t_ms = sum(a.elapsed_time(b) for a, b in ev)
    t_ms, aff_all = benchdist.reduce_time_and_work(t_ms, aff, dist, "cuda")
    if args.shard:
        aff_all = aff  # one shared graph: the work is not multiplied by the ranks
    value = aff_all / (t_ms / 1e3)

    # ---- e2e: public C ABI with HOST batches; H2D + D2H inside the timed region
    e2e = None
    if e2e_steps:
        # the caller's batches live in page-locked host memory (DMA'd straight
        # to the device by igk_step); filling them is the caller's own work
        h_batches = []
        # the step's result returns to the caller as the partition DELTA
        # (igk_partition_delta: every vertex whose part changed, P:23's
        # IGP-in-the-loop client), into a page-locked buffer
        dcap = 1 << 22
        h_delta = torch.empty((dcap, 2), dtype=torch.int32, pin_memory=True).numpy()
        pipelined = not args.shard  # igk_stage_batch / igk_step_begin / igk_step_end (single-GPU handles)
        if pipelined:  # untimed warm-up of the host-batch path (first calls size the buffers)
            G.stage_batch(batches[W + K])
            G.step_begin()
            G.step_end()
        else:
            G.step(batches[W + K])
        G.partition_delta(h_delta)
        for b in batches[W + K + 1: len(batches) - n_prof]:
            hb = torch.empty(b.shape, dtype=torch.int32, pin_memory=True).numpy()
            hb[...] = b
            h_batches.append(hb)
        torch.cuda.synchronize()
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(len(h_batches) + 1)]
        aff_e, rounds_e, dbytes = 0, 0, 0
        slab0 = G.store_stats()["slab_cap"]
        evs[0].record(stream)
        if pipelined:
            G.stage_batch(h_batches[0])
        for j, b in enumerate(h_batches):
            if pipelined:  # the H2D of batch j+1 (copy stream) overlaps step j
                G.step_begin()
                if j + 1 < len(h_batches):
                    G.stage_batch(h_batches[j + 1])
                _, st, _ = G.step_end()
            else:
                _, st, _ = G.step(b)           # igk_step: H2D DMA from pinned host memory, apply + refine
            dl = G.partition_delta(h_delta)    # D2H of the step's result: (vertex, new part) pairs
            dbytes += dl.nbytes
            aff_e += st["affected"]
            rounds_e += st["rounds"]
            evs[j + 1].record(stream)
        torch.cuda.synchronize()
        te = evs[0].elapsed_time(evs[-1])
        per = [evs[j].elapsed_time(evs[j + 1]) for j in range(len(h_batches))]
        te, aff_e = benchdist.reduce_time_and_work(te, aff_e, dist, "cuda")
        e2e = {"value": aff_e / (te / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(np.mean([b.nbytes for b in h_batches])),
               "d2h_bytes_per_step": int(dbytes / len(h_batches)),
               "d2h": "partition delta (igk_partition_delta: vertex, new part pairs); the step's ~250-byte "
                      "status head arrives through host-mapped memory",
               "api": "igk_stage_batch (H2D of batch t+1 on the copy stream) + igk_step_begin / igk_step_end "
                      "+ igk_partition_delta" if pipelined else "igk_step + igk_partition_delta",
               "ms_per_step": te / len(h_batches),
               "ms_p50": float(np.median(per)), "ms_max": float(np.max(per)),
               # the e2e steps are the iterations AFTER the device-timed ones (the graph keeps
               # changing): their work is reported so the two legs can be compared
               "affected_per_step": aff_e / len(h_batches), "rounds_per_step": rounds_e / len(h_batches),
               "store_compacted": G.store_stats()["slab_cap"] != slab0}

    # ---- per-phase roofline (profile mode, after the timed legs)
    phases = None
    if n_prof:
        pb = [torch.from_numpy(b).cuda() for b in batches[len(batches) - n_prof:]]
        phases = phase_profile(G, [(t.data_ptr(), len(t)) for t in pb], peaks()[0])

    # ---- S9 cut/weight reduction (full store scan, HBM-bound): own roofline
    s9 = None
    if not args.profile:
        t9 = []
        for _ in range(5):
            if flush is not None:
                flush.zero_()
            torch.cuda.synchronize()
            G.recount()
            t9.append(G.last_ms()["recount"])
        ss = G.store_stats()
        # algorithmic bytes (SURVEY 8(d) 2m*5 B + 16 n, made exact): every LIVE
        # entry's 4-byte ID, the 1-byte label of the neighbour for the half
        # of the entries that own the edge (x > v), and per ACTIVE vertex its
        # 16-byte record + 1-byte label
        b9 = ss["adj_entries"] * 4 + ss["adj_entries"] // 2 + ss["n_active"] * 17
        a9 = b9 / (float(np.median(t9)) / 1e3) / 1e9
        s9 = {"kernel": "k_recount3", "bound": "hbm", "achieved": a9, "unit": "GB/s", "bytes_per_launch": b9,
              "launch_ms": float(np.median(t9)), "adj_entries": ss["adj_entries"], "n_active": ss["n_active"]}

    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return
    peak, peak_kind = peaks()
    if s9:
        s9.update(peak=peak, peak_kind=peak_kind, frac=s9["achieved"] / peak)
    achieved = rbytes / (refine_ms / 1e3) / 1e9 if refine_ms > 0 else 0.0
    # batches of >= kSplitB modifiers run as k_apply + k_refine (2 launches per step)
    split = launches >= 2 * K and not args.shard
    kname = "k_apply+k_refine (split launch, one step)" if split else "k_step (apply+refine fused)"
    if args.shard:
        kname = ("k_apply x2 + k_refine_sh x5 + k_rounds_p2p (sharded step, persistent P2P rounds)" if args.p2p
                 else "k_apply x2 + k_refine_sh x(5 + 2 R) (sharded step)")
    traffic = None
    try:
        tj = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        traffic = tj.get(args.config, {}).get("k_apply+k_refine" if split else "k_step")
    except Exception:
        pass
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": W,
        "ms_per_step": t_ms / K, "higher_is_better": True, "scaling": "strong" if args.shard else "weak",
        "vs_baseline": None,
        "dtype": "int32", "data": "synthetic",
        "config": {"workload": desc, "n": g.n, "k": k,
                   "parallelism": (("sharded" + ("+p2p" if args.p2p else "")) if args.shard else "replicas")
                   if (world > 1 or args.shard) else "single",
                   "l2": "flushed between iterations (256 MiB write)" if flush is not None else "not flushed",
                   "batch_modifiers": int(np.mean([len(b) for b in batches[W:W + K]])),
                   # the stream is edge-conserving: average degree at the start of
                   # the run and after the last generated batch
                   "avg_degree_start": deg_start, "avg_degree_end": round(S.avg_degree, 3),
                   "affected_def": "|A \\ psi| + |Psi0|: placed vertices touched by the batch + pending inserts "
                                   "(R2-expanded and R3-evicted vertices are not counted: conservative)"},
        "gpu_launches": launches,
        "roofline": {"kernel": kname, "bound": "hbm", "achieved": achieved, "peak": peak,
                     "peak_kind": peak_kind, "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                     "bytes_per_launch": rbytes / K, "launch_ms": refine_ms / K,
                     "share_of_step": refine_ms / t_ms if t_ms else None},
        "kernel_ms": {kname.split(" ")[0]: refine_ms / K},
        "iteration": {"affected": aff / K, "rounds": float(np.mean([s["rounds"] for s in stats])),
                      "moves": float(np.mean([s["moves_applied"] for s in stats])),
                      "evicted": float(np.mean([s["evicted"] for s in stats])),
                      "cut_last": stats[-1]["cut"], "cap": stats[-1]["cap"],
                      "max_part_weight_last": stats[-1]["max_part_weight"], "metis_initial_cut": metis_cut,
                      "ms_p50": float(np.median([a.elapsed_time(b) for a, b in ev])),
                      "ms_p90": float(np.percentile([a.elapsed_time(b) for a, b in ev], 90))},
        "clocks": clocks,
        "roofline_s9": s9,
    }
    if e2e:
        line["e2e"] = e2e
    if phases:
        line["phases"] = phases
    if not args.no_repartition and not args.profile and not args.shard:
        line["full_repartition"] = full_repartition(G, k, G.cut(), t_ms / K)
    if not args.no_cpu_baseline and not args.profile:
        line["cpu_baseline"] = cpu_baseline(g, part, k, cfg["eps"], batches, gpu_cuts, args.cpu_iters)
    print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
