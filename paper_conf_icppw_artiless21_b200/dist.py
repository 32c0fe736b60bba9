"""Source-partitioned multi-GPU BC (north star (d)).

bc is a sum of independent per-source dependencies (Eq. 3; the source loop of
Alg. 1 l.6), so the graph is replicated on every GPU, rank r takes a contiguous range of
the source list, and ONE all-reduce(SUM) of the fp64 bc vector (NCCL over NVLink/NVSwitch)
combines them.  No other data crosses GPUs.  One process per GPU (torchrun); torch.distributed
is plumbing only -- every step of the path runs in libturbobc's kernels.
"""
from __future__ import annotations

import numpy as np


def partition(k: int, world: int, rank: int):
    """Contiguous balanced range [lo, hi) of a k-long source list for `rank` of `world`."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return k * rank // world, k * (rank + 1) // world


def _world(group):
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        return dist.get_world_size(group), dist.get_rank(group)
    return 1, 0


def shard_sum(sources, compute_partial, group=None):
    """Run compute_partial(slice) on this rank's contiguous slice of `sources` (every rank passes
    the same full list), then all-reduce(SUM) the partial vectors.  compute_partial returns a
    float64 torch tensor (zeros for an empty slice); the reduced tensor is returned."""
    import torch.distributed as dist
    world, rank = _world(group)
    lo, hi = partition(len(sources), world, rank)
    part = compute_partial(sources[lo:hi])
    if dist.is_available() and dist.is_initialized():  # also at world 1: the same collective path
        dist.all_reduce(part, op=dist.ReduceOp.SUM, group=group)
    return part


def bc_device(graph, sources, group=None, stream=None):
    """All ranks call this with the SAME full source list (torch int32, on this rank's GPU).
    Returns the all-reduced bc (torch float64 [n]) on this rank's GPU."""
    import torch

    def partial(src):
        bc = torch.zeros(graph.n, dtype=torch.float64, device=sources.device)
        if src.numel():
            graph.bc_device(src, bc, stream)
        return bc

    return shard_sum(sources, partial, group)


def bc(graph, sources, group=None) -> np.ndarray:
    """Host-to-host public entry point: numpy source list in, numpy bc out (every rank gets it).
    Copies the list H2D from pinned memory, runs this rank's slice, all-reduces, copies bc back."""
    import torch
    src = torch.from_numpy(np.ascontiguousarray(sources, dtype=np.int32)).pin_memory()
    dev = torch.device("cuda", graph.device)
    out = bc_device(graph, src.to(dev, non_blocking=True), group)
    host = torch.empty(graph.n, dtype=torch.float64).pin_memory()
    host.copy_(out, non_blocking=True)
    torch.cuda.current_stream(dev).synchronize()
    return host.numpy()
