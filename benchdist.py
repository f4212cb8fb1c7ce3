"""Multi-process plumbing of bench.py (one process per GPU, torchrun).

The refinement path itself has no data-path collective in round 1: each rank
refines its own independent graph instance ("replicas").
These helpers only (a) derive per-rank seeds and (b) reduce the per-rank
device times and work counts: time = MAX over ranks, work = SUM over ranks.
They run on NCCL on the GPU box and on gloo in the CPU tests.
"""
from __future__ import annotations

import os

import igk_inputs as gi


def env_ranks():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def rank_graph_seed(cfg_index: int, rank: int) -> int:
    """rank 0 gets the canonical BASELINE seed; others an offset instance"""
    return gi.graph_seed(cfg_index) + 1000 * rank


def reduce_time_and_work(t_ms: float, work: float, dist=None, device="cpu"):
    """(max over ranks of t_ms, sum over ranks of work); identity without dist."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(t_ms), float(work)
    import torch
    if dist.get_backend() == "gloo":
        device = "cpu"
    t = torch.tensor([float(t_ms)], dtype=torch.float64, device=device)
    w = torch.tensor([float(work)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dist.all_reduce(w, op=dist.ReduceOp.SUM)
    return t.item(), w.item()
