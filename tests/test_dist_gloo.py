"""Host logic of the multi-GPU source batch (sharding + gather order), on CPU
with world_size 2 gloo processes (the GPU path uses the same code over NCCL)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icppw_zhangczsdhay23_b200 import batch


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n_sources, V, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    mine = batch.shard_sources(np.arange(n_sources) * 10, rank, world)
    # fake distance rows: row for global source i holds i*1000 + column
    rows = torch.stack([torch.arange(V, dtype=torch.int32) + int(s // 10) * 1000 for s in mine]) if len(mine) \
        else torch.zeros((0, V), dtype=torch.int32)
    out = batch.gather_rows(rows, n_sources, dst=0)
    if rank == 0:
        q.put(out.numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("n_sources", [64, 7])
def test_gather_two_ranks(n_sources):
    world, V = 2, 13
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_sources, V, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    exp = np.stack([np.arange(V) + i * 1000 for i in range(n_sources)]).astype(np.int32)
    assert np.array_equal(got, exp)


def test_shard_and_order():
    src = np.arange(64)
    shards = [batch.shard_sources(src, r, 8) for r in range(8)]
    assert sorted(np.concatenate(shards).tolist()) == src.tolist()
    order = batch.global_order(64, 8)
    for r in range(8):
        assert (order[r] == shards[r]).all()
    o = batch.global_order(7, 2)
    assert o.tolist() == [[0, 2, 4, 6], [1, 3, 5, -1]]
