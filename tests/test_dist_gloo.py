"""N>1 plumbing of bench.py on CPU: world_size 2 over gloo (127.0.0.1).
Each rank gets its own graph instance (replicas); the reduction gives every
rank the max device time and the summed work."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import benchdist
    import igk_inputs as gi
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r, w, lr = benchdist.env_ranks()
    seed = benchdist.rank_graph_seed(2, r)
    g = gi.make_graph(2000, 64, seed)
    t, work = benchdist.reduce_time_and_work(1.5 + r, 10.0 * (r + 1), dist)
    q.put((r, w, seed, int(g.xadj[-1]), t, work))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_replicas_gloo():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert [r[1] for r in res] == [2, 2]
    assert res[0][2] != res[1][2]             # distinct replica seeds
    assert res[0][3] != res[1][3]             # distinct graphs
    assert res[0][4] == res[1][4] == 2.5      # max of the rank times
    assert res[0][5] == res[1][5] == 30.0     # sum of the rank work


def test_single_process_identity():
    import benchdist
    assert benchdist.reduce_time_and_work(3.0, 7, None) == (3.0, 7.0)
