"""Host logic of the multi-GPU source batch (block sharding, grouped gather
straight into the global order, §8(e) overlap), on CPU with world_size 2 gloo
processes (the GPU path uses the same code over NCCL)."""
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


class FakeGraph:
    """Stands in for a Graph: 'distance rows' are source * 1000 + column; records the calls."""

    def __init__(self, V):
        self.V, self.f32, self.torch_device, self.calls = V, False, "cpu", []

    def _fill(self, srcs, delta, out, ld):
        self.calls.append(len(srcs))
        for i, s in enumerate(srcs):
            out[i] = torch.arange(self.V, dtype=torch.int32) + int(s) * 1000

    run_multi = run_batch = _fill


def _worker(rank, world, port, n_sources, V, mode, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    sources = np.arange(n_sources) * 3 + 1
    if mode == "gather":
        mine = batch.shard_sources(sources, rank, world)
        rows = torch.stack([torch.arange(V, dtype=torch.int32) + int(s) * 1000 for s in mine]) if len(mine) \
            else torch.zeros((0, V), dtype=torch.int32)
        out = batch.gather_rows(rows, n_sources, dst=0)
        calls = []
    else:
        G = FakeGraph(V)
        out = batch.run_sharded(G, sources, 16, dst=0, kernel=mode, group_size=5)
        calls = G.calls
    q.put((rank, None if out is None else out.numpy(), calls))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("n_sources", [64, 7, 1])
@pytest.mark.parametrize("mode", ["gather", "multi", "per_source"])
def test_gather_two_ranks(n_sources, mode):
    world, V = 2, 13
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_sources, V, mode, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r, out, calls = q.get(timeout=120)
        res[r] = (out, calls)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    sources = np.arange(n_sources) * 3 + 1
    exp = np.stack([np.arange(V) + s * 1000 for s in sources]).astype(np.int32)
    assert res[1][0] is None
    assert np.array_equal(res[0][0], exp)
    if mode != "gather":  # groups of <= 5 sources, in order, covering each rank's block
        for r in range(world):
            lo, hi, _ = batch.shard_bounds(n_sources, r, world)
            assert sum(res[r][1]) == hi - lo and all(c <= 5 for c in res[r][1])


def test_shard_bounds():
    for n in (64, 7, 1, 0):
        for world in (1, 2, 4, 8):
            got = np.concatenate([batch.shard_sources(np.arange(n), r, world) for r in range(world)])
            assert got.tolist() == list(range(n))  # blocks, in order: gathered layout = global order
            k = batch.shard_bounds(n, 0, world)[2]
            assert all(len(batch.shard_sources(np.arange(n), r, world)) <= k for r in range(world))
