"""Multi-process (world_size 2, gloo, CPU) tests of the sharding / gather
host logic used for multi-GPU runs."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_cgo_sommera022_b200.parallel import (shard_range, shard_sizes, gather_results,
                                                     gather_into, sharded_infer)


def test_shard_ranges_cover_exactly_once():
    for n in (0, 1, 7, 100, 1_000_003):
        for world in (1, 2, 3, 4, 8):
            rs = [shard_range(n, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
            sz = shard_sizes(n, world)
            assert max(sz) - min(sz) <= 1 and sum(sz) == n


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class _FakePlan:
    """Stands in for a GPU Plan: a per-sample function of the features, so
    the test checks shard boundaries and gather order, not the kernels."""
    def infer(self, x, marginal=False):
        out = (x.double().sum(1, keepdim=True) * (2 if marginal else 1)).float()
        am = torch.argmax(x, dim=1).to(torch.int32)
        return out, am


def _worker(rank, world, port, n, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = torch.Generator().manual_seed(0)
        x = torch.randn((n, 5), generator=g)
        out, am = sharded_infer(_FakePlan(), x, marginal=True, gather=True)
        ref_out, ref_am = _FakePlan().infer(x, marginal=True)
        ok = torch.equal(out, ref_out) and torch.equal(am, ref_am)
        lo, hi = shard_range(n, rank, world)
        loc = torch.arange(lo, hi, dtype=torch.int64)
        full = gather_results(loc, n)
        ok = ok and torch.equal(full, torch.arange(n, dtype=torch.int64))
        # the bench's strong-scaling gather: equal shards into a preallocated buffer
        m = n - n % world
        a, b = shard_range(m, rank, world)
        logp = torch.stack([torch.arange(a, b, dtype=torch.float32)] * 3, dim=1)
        buf = torch.empty((m, 3), dtype=torch.float32)
        gather_into(buf, logp)
        ok = ok and torch.equal(buf[:, 0], torch.arange(m, dtype=torch.float32))
        am_buf = torch.empty((m,), dtype=torch.int32)
        gather_into(am_buf, torch.arange(a, b, dtype=torch.int32))
        ok = ok and torch.equal(am_buf, torch.arange(m, dtype=torch.int32))
        q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n", [10, 1001])
def test_gather_world2_gloo(n):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert sorted(res) == [(0, True), (1, True)]
