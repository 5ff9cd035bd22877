"""Multi-source batch across GPUs (north star: "a batch of independent sources
is spread across the 8xB200 box: each GPU holds a replicated graph, and NCCL
gathers distance vectors over NVLink").

One process per GPU (torchrun). Sources are sharded in contiguous blocks
(rank r gets sources [r*k, (r+1)*k), k = ceil(n / world)), so the gathered
layout [world, k, V] IS the global source order: rank ``dst`` hands NCCL
views of one [world*k, V] output tensor and never reorders or copies rows.

Fusion (§8(e)): every rank computes its shard in groups of up to 32 sources
(one ``sssp_run_multi`` launch, or ``sssp_run_batch`` runs, per group) and
starts the gather of a group's rows (``dist.gather(async_op=True)``, NCCL's
own stream) as soon as the library returns them, while the next group
computes -- the transfer of group g overlaps the SSSPs of group g+1. The
library reports run errors per call (sssp.h "Run errors"), so a failed group
raises before its rows are sent.
"""
from __future__ import annotations

import numpy as np

GROUP = 32  # sources per sssp_run_multi launch (the kernel's lane count)


def shard_bounds(n: int, rank: int, world: int):
    """Block shard of n sources: (first, end, k) with k = ceil(n / world) rows per rank."""
    k = (n + world - 1) // world
    lo = min(n, rank * k)
    return lo, min(n, lo + k), k


def shard_sources(sources, rank: int, world: int):
    """Contiguous block of the global source list owned by ``rank``."""
    lo, hi, _ = shard_bounds(len(sources), rank, world)
    return np.asarray(sources)[lo:hi]


def _gather(send, out, first: int, count: int, k: int, dst: int, group, async_op: bool):
    """Gather rows [first, first+count) of every rank's k-row shard into ``out`` on dst:
    rank r's rows land in out[r*k + first : r*k + first + count] (views, no copies)."""
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    gl = [out[r * k + first: r * k + first + count] for r in range(world)] if rank == dst else None
    return dist.gather(send[first: first + count], gl, dst=dst, group=group, async_op=async_op)


def gather_rows(local_rows, n_sources: int, dst: int = 0, group=None, out=None):
    """Gather every rank's block of rows (``local_rows`` [len(shard), V]) to ``dst``.

    Returns [n_sources, V] on ``dst`` (a view of ``out`` if given, shape
    [world*k, V]) and None elsewhere. Shorter shards (only the last ranks when
    world does not divide n) are padded on the send side only."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    _, _, k = shard_bounds(n_sources, rank, world)
    V = local_rows.shape[1]
    send = local_rows
    if send.shape[0] != k:
        send = torch.zeros((k, V), dtype=local_rows.dtype, device=local_rows.device)
        send[: local_rows.shape[0]] = local_rows
    if rank == dst and out is None:
        out = torch.empty((world * k, V), dtype=local_rows.dtype, device=local_rows.device)
    if k:
        _gather(send.contiguous(), out, 0, k, k, dst, group, async_op=False)
    return out[:n_sources] if rank == dst else None


def run_sharded(graph, sources, delta, dst: int = 0, group=None, kernel: str = "multi", out=None,
                group_size: int = GROUP, on_group=None):
    """Run this rank's block of ``sources`` on ``graph`` (a Graph on this rank's
    GPU) and gather all distance rows to ``dst``, overlapping each group's
    gather with the next group's compute. ``kernel``: "multi" = 32 sources per
    persistent launch (``sssp_run_multi``, NEXT-4), "per_source" = one
    Delta-stepping launch per source (``sssp_run_batch``). Identical rows.
    ``on_group(first, count, work)`` (dst only) is called once group rows
    [r*k + first, r*k + first + count) of every rank r have been enqueued into
    ``out`` (``work``: the async gather, or None without a process group), so a
    caller can stream them onward (e.g. D2H) while the next group computes.
    Without an initialised process group this is the single-GPU case: the rows
    are computed straight into ``out``.
    Returns [len(sources), V] on ``dst`` (in global source order), else None."""
    import torch
    import torch.distributed as dist

    if kernel not in ("per_source", "multi"):
        raise ValueError(f"unknown kernel {kernel!r}")
    n = len(sources)
    run = graph.run_multi if kernel == "multi" else graph.run_batch
    if not (dist.is_available() and dist.is_initialized()):
        dev = getattr(graph, "torch_device", None) or f"cuda:{graph.device}"
        if out is None:
            out = torch.empty((max(n, 1), graph.V), dtype=torch.float32 if graph.f32 else torch.int32, device=dev)
        src = np.asarray(sources)
        for g0 in range(0, n, group_size):
            cnt = min(group_size, n - g0)
            run(src[g0: g0 + cnt], delta, out[g0: g0 + cnt], graph.V)
            if on_group is not None:
                on_group(g0, cnt, None)
        return out[:n]
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    lo, hi, k = shard_bounds(n, rank, world)
    mine = np.asarray(sources)[lo:hi]
    dev = getattr(graph, "torch_device", None) or f"cuda:{graph.device}"
    dtype = torch.float32 if graph.f32 else torch.int32
    staged = dist.get_backend(group) != "nccl" and str(dev).startswith("cuda")  # gloo: host buffers (tests)
    send = torch.empty((max(k, 1), graph.V), dtype=dtype, device=dev)
    send_h = torch.zeros((max(k, 1), graph.V), dtype=dtype) if staged else None
    if rank == dst and out is None:
        out = torch.empty((world * k, graph.V), dtype=dtype, device="cpu" if staged else dev)
    works = []
    for g0 in range(0, k, group_size):
        cnt = min(group_size, k - g0)
        real = max(0, min(cnt, len(mine) - g0))
        if real:
            run(mine[g0: g0 + real], delta, send[g0: g0 + real], graph.V)  # returns when the rows are done
        buf = send
        if staged:
            send_h[g0: g0 + cnt] = send[g0: g0 + cnt].cpu()
            buf = send_h
        works.append(_gather(buf, out, g0, cnt, k, dst, group, async_op=True))
        if on_group is not None and rank == dst:
            on_group(g0, cnt, works[-1])
    for w in works:
        w.wait()
    if rank != dst:
        return None
    return out[:n]
