"""Sharded refinement (igk_refine_sharded): the round gain is split by owner
and the move records are all-gathered every round.

* CPU (`-m "not gpu"`): the record exchange itself (TorchComm over gloo,
  world_size 2 and 3, uneven contributions) concatenates in rank order.
* GPU: 2 and 3 ranks (processes) sharing the one test GPU, gloo for the
  exchange; every rank's partition, cut and stats must equal the oracle's
  (and each other's) on every iteration of a C1 stream and a weighted stream.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


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


def _exchange_worker(rank, world, port, q):
    dist = _init(rank, world, port)
    import paper_conf_dac_leejlczcshh25_b200 as igk
    comm = igk.TorchComm()
    mine = np.arange(4 * (rank + 1), dtype=np.int32).reshape(-1, 4) + 1000 * rank
    out = comm.gather_records(mine)
    empty = comm.gather_records(np.zeros((0, 4), np.int32))
    q.put((rank, out.tolist(), len(empty)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_record_allgather_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_exchange_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    expect = np.concatenate([np.arange(4 * (r + 1), dtype=np.int32).reshape(-1, 4) + 1000 * r
                             for r in range(world)]).tolist()
    for r, out, ne in res:
        assert out == expect and ne == 0


def _shard_worker(rank, world, port, q, weighted):
    dist = _init(rank, world, port)
    import torch
    torch.cuda.set_device(0)
    import igk_inputs as gi
    import paper_conf_dac_leejlczcshh25_b200 as igk
    n, k = 10_000, 4
    g = gi.make_graph(n, 64, gi.graph_seed(1), weighted=weighted)
    part, _ = gi.metis_partition(g, k)
    G = igk.IGKGraph(g.xadj, g.adjncy, k, 0.03, part, g.vwgt, g.adjwgt)
    comm = igk.TorchComm()
    O = None
    if rank == 0:
        import oracle
        O = oracle.Oracle(g.xadj, g.adjncy, k, 0.03, part, g.vwgt, g.adjwgt)
    S = gi.Stream(g, 77, weighted=weighted)
    log = []
    st0 = G.refine_sharded(comm)[1]
    if O is not None:
        O.refine()
    for it in range(8):
        b = S.next(gi.MODE_MIX, 0.03)
        assert G.apply(b)[0] == 0
        _, st = G.refine_sharded(comm)
        p = G.partition()
        entry = {"it": it, "part": p.tobytes(), "cut": G.cut(), "recount": G.recount()[0], "stats": st}
        if O is not None:
            O.apply(b)
            _, so = O.refine()
            entry["oracle_part"] = O.partition().tobytes()
            entry["oracle_stats"] = so
        log.append(entry)
    q.put((rank, log, comm.calls))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("world,weighted", [(2, False), (3, True)])
def test_sharded_refine_matches_oracle(world, weighted):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_shard_worker, args=(r, world, port, q, weighted)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted((q.get(timeout=600) for _ in range(world)), key=lambda t: t[0])
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    logs = [r[1] for r in res]
    assert all(r[2] > 0 for r in res)  # rounds really exchanged records
    common = ["affected", "inserted", "expanded", "filtered_in", "expanded_in", "evicted", "rounds",
              "moves_applied", "moves_deferred", "cut", "cap", "max_part_weight", "imbalanced"]
    for it in range(len(logs[0])):
        e0 = logs[0][it]
        assert e0["part"] == e0["oracle_part"], f"rank 0 vs oracle at iteration {it}"
        assert all(e0["stats"][f] == e0["oracle_stats"][f] for f in common), it
        assert e0["cut"] == e0["recount"]
        for lg in logs[1:]:
            assert lg[it]["part"] == e0["part"] and lg[it]["cut"] == e0["cut"]
