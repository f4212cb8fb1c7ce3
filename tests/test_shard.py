"""Vertex-range sharded handles.

Rank r of N owns a range of vertex IDs, stores their adjacency plus the
ghost prefixes pointing at them, and keeps labels / weights / W_p
replicated; every refine exchanges fixed-size all-reduces (the R1 / R2
candidate bitmaps, the restoration keys, the per-round move records of the
selected vertices).  Results must be bit-identical to one GPU and
to the oracle.

* CPU (`-m "not gpu"`): the host-callback transport (TorchComm over gloo,
  world 2 and 3) -- SUM of disjoint bit patterns (the bitmap OR, incl. the
  sign bit), MIN / MAX, uint32 records with the high bit set.
* GPU: 2 and 3 ranks (processes) sharing the test GPU over gloo: every
  rank's partition, cut, W_p and stats equal the oracle's on every iteration
  of a C1 stream (check mode: the collective recount), a weighted stream, an
  adversarial stream (restoration fires: keys all-reduced), a hub graph, and
  through igk_step with an invalid batch (rejected on every rank alike).
* GPU, NCCL: the protocol with ONE rank over a real NCCL communicator
  (loopback) created inside the library from igk_nccl_unique_id.
"""
import ctypes as C
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

COMMON = ["affected", "inserted", "expanded", "filtered_in", "expanded_in", "evicted", "rounds",
          "moves_applied", "moves_deferred", "cut", "cap", "max_part_weight", "imbalanced"]


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    return dist


def _spawn(target, world, *args, timeout=900):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=target, args=(r, world, port, q) + args) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted((q.get(timeout=timeout) for _ in range(world)), key=lambda t: t[0])
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    return res


# ---------------------------------------------------------------------------
# CPU: the transport
# ---------------------------------------------------------------------------
def _xp_worker(rank, world, port, q):
    dist = _init(rank, world, port)
    import paper_conf_dac_leejlczcshh25_b200 as igk
    comm = igk.TorchComm()
    out = {}
    # bitmap OR as a SUM of disjoint bits (bit 63 included): rank r owns bits r, r + world, ...
    bm = np.zeros(4, np.uint64)
    for b in range(rank, 256, world):
        bm[b // 64] |= np.uint64(1) << np.uint64(b % 64)
    bmi = bm.view(np.int64).copy()
    assert comm._allreduce(None, bmi.ctypes.data, 4, 0, 0) == 0
    out["bitmap"] = bmi.view(np.uint64).tolist()
    v = np.array([10 + rank, -5 * rank], np.int64)
    assert comm._allreduce(None, v.ctypes.data, 2, 0, 1) == 0
    out["min"] = v.tolist()
    v = np.array([10 + rank, -5 * rank], np.int64)
    assert comm._allreduce(None, v.ctypes.data, 2, 0, 2) == 0
    out["max"] = v.tolist()
    r = np.zeros(3 * world, np.uint32)  # records: position j written by rank j % world only
    for j in range(rank, 3 * world, world):
        r[j] = 0x80000000 + j
    assert comm._allreduce(None, r.ctypes.data, len(r), 1, 0) == 0
    out["u32"] = r.tolist()
    q.put((rank, out))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_transport_allreduce_gloo(world):
    res = _spawn(_xp_worker, world, timeout=120)
    for _, out in res:
        assert out["bitmap"] == [0xFFFFFFFFFFFFFFFF] * 4
        assert out["min"] == [10, -5 * (world - 1)]
        assert out["max"] == [10 + world - 1, 0]
        assert out["u32"] == [0x80000000 + j for j in range(3 * world)]


# ---------------------------------------------------------------------------
# GPU: sharded handles vs the oracle
# ---------------------------------------------------------------------------
def _scenario(name):
    import igk_inputs as gi
    if name == "C1":
        g = gi.make_graph(10_000, 64, gi.graph_seed(1))
        part, _ = gi.metis_partition(g, 4)
        return g, part, 4, 0.03, gi.Stream(g, 77), dict(mode=gi.MODE_MIX, frac=0.03, iters=8, check=True)
    if name == "weighted":
        g = gi.make_graph(20_000, 256, 991, weighted=True)
        part, _ = gi.metis_partition(g, 8)
        return g, part, 8, 0.03, gi.Stream(g, 78, weighted=True), dict(mode=gi.MODE_MIX, frac=0.05, iters=6,
                                                                         check=False)
    if name == "adversarial":
        g = gi.make_graph(40_000, 1000, gi.graph_seed(5))
        part, _ = gi.metis_partition(g, 8)
        S = gi.Stream(g, 79, region0=(part == 0).astype(np.int32))
        return g, part, 8, 0.03, S, dict(mode=gi.MODE_ADVERSARIAL, nvd=400, nvi=200, iters=10, check=False)
    raise ValueError(name)


def _hub_graph():
    import igk_inputs as gi
    rng = np.random.default_rng(9)
    n = 6000
    edges = {(u, u + 1) for u in range(n - 1)}
    for h in (100, 3100):
        for v in rng.choice(np.arange(n), size=1500, replace=False):
            if int(v) != h:
                edges.add((min(h, int(v)), max(h, int(v))))
    adj = {u: set() for u in range(n)}
    for a, b in edges:
        adj[a].add(b)
        adj[b].add(a)
    xadj, a = [0], []
    for u in range(n):
        a += sorted(adj[u])
        xadj.append(len(a))
    return gi.Graph(np.array(xadj, np.int64), np.array(a, np.int32), None, None)


def _shard_worker(rank, world, port, q, name):
    dist = _init(rank, world, port)
    import torch
    torch.cuda.set_device(0)
    import igk_inputs as gi
    import oracle
    import paper_conf_dac_leejlczcshh25_b200 as igk
    comm = igk.TorchComm()
    if name == "hub":
        g = _hub_graph()
        part = gi.block_partition(g.n, 2)
        k, eps, S, cfg = 2, 0.5, gi.Stream(g, 80), dict(mode=gi.MODE_MIX, frac=0.05, iters=6, check=True)
    else:
        g, part, k, eps, S, cfg = _scenario(name)
    G = igk.IGKGraph(g.xadj, g.adjncy, k, eps, part, g.vwgt, g.adjwgt, check=cfg["check"],
                     nranks=world, rank=rank, comm=comm)
    O = oracle.Oracle(g.xadj, g.adjncy, k, eps, part, g.vwgt, g.adjwgt) if rank == 0 else None
    log = []

    def record(tag, st):
        e = {"tag": tag, "part": G.partition().tobytes(), "cut": G.cut(), "wp": G.part_weights().tolist(),
             "stats": {f: st[f] for f in COMMON}, "delta": sorted(map(tuple, G.partition_delta().tolist()))}
        if O is not None:
            e["o_part"] = O.partition().tobytes()
            e["o_cut"] = O.cut()
            e["o_wp"] = O.part_weights().tolist()
        return e

    _, st = G.refine()
    if O is not None:
        O.refine()
    log.append(record("settle", st))
    for it in range(cfg["iters"]):
        if cfg["mode"] == gi.MODE_ADVERSARIAL:
            b = S.next(cfg["mode"], 0.0, cfg["nvd"], cfg["nvi"], 0, 0)
        else:
            b = S.next(cfg["mode"], cfg["frac"])
        if name == "C1" and it % 2:  # igk_step (apply + refine, both collective)
            s, st, bad = G.step(b)
            assert s in (igk.OK, igk.WIMBALANCED) and bad == -1
        else:
            s, fid, bad = G.apply(b)
            assert s == igk.OK, (s, bad)
            _, st = G.refine()
        e = record(f"it{it}", st)
        if O is not None:
            assert O.apply(b)[0] == 0
            pre = O.partition()
            _, so = O.refine()
            e["o_part"] = O.partition().tobytes()
            e["o_cut"] = O.cut()
            e["o_wp"] = O.part_weights().tolist()
            e["o_stats"] = {f: so[f] for f in COMMON}
            post = O.partition()
            old = np.full(len(post), -2, np.int32)
            old[: len(pre)] = pre
            idx = np.nonzero((post >= 0) & (post != old))[0]
            e["o_delta"] = sorted(zip(idx.tolist(), post[idx].tolist()))
            inv = O.check_invariants(e["cut"])
            assert inv is None, inv
        log.append(e)
    # an invalid batch (self loop) is rejected on every rank, nothing changes
    if name == "C1":
        before = (G.partition().tobytes(), G.cut())
        s, st, bad = G.step(np.array([[3, 5, 5, 1]], np.int32))
        assert s == igk.EINVAL and bad == 0
        assert (G.partition().tobytes(), G.cut()) == before
    q.put((rank, log, comm.calls))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("world,name", [(2, "C1"), (3, "C1"), (2, "weighted"), (3, "adversarial"), (2, "hub")])
def test_sharded_matches_oracle(world, name):
    res = _spawn(_shard_worker, world, name)
    logs = [r[1] for r in res]
    assert all(r[2] > 0 for r in res)  # the ranks really exchanged
    for i, e0 in enumerate(logs[0]):
        where = f"{name} world {world} {e0['tag']}"
        assert e0["part"] == e0["o_part"], where
        assert e0["cut"] == e0["o_cut"] and e0["wp"] == e0["o_wp"], where
        if "o_stats" in e0:
            diff = {f: (e0["o_stats"][f], e0["stats"][f]) for f in COMMON if e0["o_stats"][f] != e0["stats"][f]}
            assert not diff, (where, diff)
            assert e0["delta"] == [tuple(x) for x in e0["o_delta"]], where
        for lg in logs[1:]:
            assert lg[i]["part"] == e0["part"] and lg[i]["cut"] == e0["cut"], where
            assert lg[i]["stats"] == e0["stats"] and lg[i]["delta"] == e0["delta"], where
    if name == "adversarial":
        assert sum(e["stats"]["evicted"] for e in logs[0]) > 0


@pytest.mark.gpu
def test_sharded_protocol_over_nccl_one_rank():
    """The sharded protocol (staged launches, bitmaps, canonical pending list,
    per-round records) through a real NCCL communicator created inside the
    library (one rank, loopback), bit-exact with the oracle on a C1 stream."""
    import igk_inputs as gi
    from tests.parity import Pair
    import paper_conf_dac_leejlczcshh25_b200 as igk
    g = gi.make_graph(10_000, 64, gi.graph_seed(1))
    part, _ = gi.metis_partition(g, 4)
    uid = igk.nccl_unique_id()
    assert len(uid) == 128
    P = Pair(g.xadj, g.adjncy, 4, 0.03, part, check=True, nranks=1, rank=0, nccl_id=uid)
    P.refine("settle")
    S = gi.Stream(g, 81)
    for it in range(6):
        assert P.apply(S.next(gi.MODE_MIX, 0.03), f"it{it}") == 0
        P.refine(f"it{it}")
        P.compare_state(f"it{it}", full_csr=(it == 5))


# ---------------------------------------------------------------------------
# NEXT-3: persistent P2P round kernel (records through peer memory, device
# barrier).  N ranks as N threads of ONE process sharing the test GPU: each
# rank's persistent kernel takes 1/N of the SMs so all are resident at once;
# peers are plain device pointers (the same code maps CUDA IPC handles when
# the ranks are processes on different GPUs).  The host collectives of the
# pre-round phases go through an in-process transport.
# ---------------------------------------------------------------------------
class _ThreadComm:
    """igk_comm for N threads of one process: all-reduce through a shared
    numpy buffer and a barrier (test transport; the library calls it from
    each rank's thread, ctypes holds the GIL only inside the callback)."""

    def __init__(self, n):
        import threading
        import paper_conf_dac_leejlczcshh25_b200 as igk
        self.n = n
        self.bar = threading.Barrier(n)
        self.slots = [None] * n
        self.out = None
        self.structs = []
        self.cbs = []
        for r in range(n):
            cb = igk.ALLREDUCE_FN(lambda ctx, buf, count, dtype, op, r=r: self._ar(r, buf, count, dtype, op))
            self.cbs.append(cb)
            self.structs.append(igk.Comm(None, cb))

    def _ar(self, r, buf, count, dtype, op):
        try:
            name, size = {0: ("int64", 8), 1: ("uint32", 4)}[dtype]
            arr = np.ctypeslib.as_array((C.c_uint8 * (count * size)).from_address(buf)).view(name)
            self.slots[r] = arr.astype(np.int64)
            self.bar.wait()
            if r == 0:
                st = np.stack(self.slots)
                self.out = st.sum(0) if op == 0 else (st.min(0) if op == 1 else st.max(0))
            self.bar.wait()
            arr[:] = self.out.astype(name)
            self.bar.wait()
            return 0
        except Exception:
            import traceback
            traceback.print_exc()
            return -1


class _CommRef:
    def __init__(self, struct):
        self.struct = struct


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
def test_p2p_rounds_match_oracle(world):
    import threading
    import igk_inputs as gi
    import oracle
    import paper_conf_dac_leejlczcshh25_b200 as igk
    g = gi.make_graph(10_000, 64, gi.graph_seed(1))
    part, _ = gi.metis_partition(g, 4)
    S = gi.Stream(g, 82)
    batches = [S.next(gi.MODE_MIX, 0.03) for _ in range(8)]
    O = oracle.Oracle(g.xadj, g.adjncy, 4, 0.03, part)
    O.refine()
    expect = []
    for b in batches:
        assert O.apply(b)[0] == 0
        _, so = O.refine()
        expect.append((O.partition().tobytes(), so["cut"], so["rounds"], so["moves_applied"]))
    tc = _ThreadComm(world)
    res = [None] * world
    err = [None] * world

    def run(r):
        try:
            import torch
            stream = torch.cuda.Stream()  # one non-blocking stream per rank: the persistent kernels run side by side
            G = igk.IGKGraph(g.xadj, g.adjncy, 4, 0.03, part, nranks=world, rank=r, stream=stream.cuda_stream,
                             comm=_CommRef(tc.structs[r]), p2p=True, ranks_per_device=world, check=True)
            G.refine()
            out = []
            for b in batches:
                s, _, bad = G.apply(b)
                assert s == 0, (s, bad)
                _, st = G.refine()
                out.append((G.partition().tobytes(), G.cut(), st["rounds"], st["moves_applied"]))
            res[r] = (out, G.debug_paths())
            G.close()
        except Exception as e:  # reported by the main thread
            import traceback
            err[r] = traceback.format_exc()

    ts = [threading.Thread(target=run, args=(r,)) for r in range(world)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=600)
    assert not any(err), err
    for r in range(world):
        for it, (got, exp) in enumerate(zip(res[r][0], expect)):
            assert got == exp, (r, it)
