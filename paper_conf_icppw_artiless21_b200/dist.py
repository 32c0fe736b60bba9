"""Source-partitioned multi-GPU BC (north star (d)).

bc is a sum of independent per-source dependencies (Eq. 3; the source loop of Alg.1 l.6,
P:122), so the graph is replicated on every GPU, rank r takes a contiguous range of the source
list, and ONE all-reduce(SUM) of the fp64 bc vector (NCCL over NVLink/NVSwitch) combines them.
No other data crosses GPUs.  One process per GPU (torchrun), ``torch.distributed`` plumbing.
"""
from __future__ import annotations

import numpy as np


def partition(k: int, world: int, rank: int):
    """Contiguous balanced range [lo, hi) of a k-long source list for `rank` of `world`."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return k * rank // world, k * (rank + 1) // world


def bc_device(graph, sources, group=None, stream=None):
    """All ranks call this with the SAME full source list (torch int32, on this rank's GPU).
    Returns the all-reduced bc (torch float64 [n]) on this rank's GPU."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    lo, hi = partition(sources.numel(), world, rank)
    bc = torch.zeros(graph.n, dtype=torch.float64, device=sources.device)
    if hi > lo:
        graph.bc_device(sources[lo:hi], bc, stream)
    if world > 1:
        dist.all_reduce(bc, op=dist.ReduceOp.SUM, group=group)
    return bc


def bc(graph, sources, group=None) -> np.ndarray:
    """Host-to-host public entry point: numpy source list in, numpy bc out (every rank gets it).
    Copies this rank's slice H2D from pinned memory, runs, all-reduces, copies bc back."""
    import torch
    src = torch.from_numpy(np.ascontiguousarray(sources, dtype=np.int32)).pin_memory()
    dev = torch.device("cuda", graph.device)
    out = bc_device(graph, src.to(dev, non_blocking=True), group)
    host = torch.empty(graph.n, dtype=torch.float64).pin_memory()
    host.copy_(out, non_blocking=True)
    torch.cuda.current_stream(dev).synchronize()
    return host.numpy()


def reduce_partials(partials_by_rank):
    """Host-side model of the reduction (used by CPU tests of the partition logic)."""
    return np.sum(np.stack(partials_by_rank), axis=0)
