"""Multi-source batch across GPUs (north star: "a batch of independent sources
is spread across the 8xB200 box: each GPU holds a replicated graph, and NCCL
gathers distance vectors over NVLink").

One process per GPU (torchrun). Sources are sharded round-robin
(``sources[rank::world]``); every rank runs its shard through the C-ABI
(``sssp_run_batch`` writes rows straight into a device tensor), then the rows
are gathered to the destination rank with one ``torch.distributed`` gather
(NCCL on GPUs; gloo for the CPU tests of this host logic).
"""
from __future__ import annotations

import numpy as np


def shard_sources(sources, rank: int, world: int):
    """Round-robin shard: global source i goes to rank i % world, row i // world."""
    return np.asarray(sources)[rank::world]


def global_order(n: int, world: int):
    """Gather layout -> global source index: gathered[r][j] is source r + j*world."""
    k = (n + world - 1) // world
    idx = np.full((world, k), -1, dtype=np.int64)
    for i in range(n):
        idx[i % world, i // world] = i
    return idx


def gather_rows(local_rows, n_sources: int, dst: int = 0, group=None):
    """Gather every rank's [k_r, V] rows to ``dst`` in global source order.

    local_rows: tensor [k_r, V] (k_r = shard size of this rank; shards differ by
    at most one row and are zero-padded to the largest for the collective).
    Returns [n_sources, V] on ``dst`` and None elsewhere."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    k = (n_sources + world - 1) // world
    V = local_rows.shape[1]
    if local_rows.shape[0] < k:
        pad = torch.zeros((k - local_rows.shape[0], V), dtype=local_rows.dtype, device=local_rows.device)
        local_rows = torch.cat([local_rows, pad], 0)
    local_rows = local_rows.contiguous()
    if dist.get_backend(group) != "nccl" and local_rows.is_cuda:  # gloo: host staging (tests)
        local_rows = local_rows.cpu()
    bufs = [torch.empty_like(local_rows) for _ in range(world)] if rank == dst else None
    dist.gather(local_rows, bufs, dst=dst, group=group)
    if rank != dst:
        return None
    order = global_order(n_sources, world)
    out = torch.empty((n_sources, V), dtype=local_rows.dtype, device=local_rows.device)
    for r in range(world):
        for j in range(k):
            i = order[r, j]
            if i >= 0:
                out[i] = bufs[r][j]
    return out


def run_sharded(graph, sources, delta, dst: int = 0, group=None, kernel: str = "per_source"):
    """Run this rank's shard of ``sources`` on ``graph`` (a paper_conf...Graph on
    this rank's GPU) and gather all distance rows to ``dst``. ``kernel``:
    "per_source" = one persistent Delta-stepping launch per source
    (``sssp_run_batch``), "multi" = 32 sources per launch (``sssp_run_multi``,
    NEXT-4). Both give identical rows."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    mine = shard_sources(sources, rank, world)
    dtype = torch.float32 if graph.f32 else torch.int32
    rows = torch.empty((max(len(mine), 1), graph.V), dtype=dtype, device=f"cuda:{graph.device}")
    if kernel not in ("per_source", "multi"):
        raise ValueError(f"unknown kernel {kernel!r}")
    if len(mine):
        (graph.run_multi if kernel == "multi" else graph.run_batch)(mine, delta, rows, graph.V)
    torch.cuda.synchronize(graph.device)
    return gather_rows(rows[: len(mine)] if len(mine) else rows[:0], len(sources), dst, group)
