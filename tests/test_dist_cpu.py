"""Multi-process host logic of the batch-sharded chain
on CPU with gloo, world size 2: shard ranges cover the batch exactly once,
the output all-gather reassembles the per-rank shards in rank order, the
max-over-ranks timing reduction, and per-image independence (O8): running
shards separately equals running the whole batch."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import dist as D


def test_shard_ranges_partition_the_batch():
    for N in (1, 7, 32, 256, 255):
        for world in (1, 2, 3, 4, 8):
            covered = []
            for r in range(world):
                lo, hi = D.shard_range(N, r, world)
                covered.extend(range(lo, hi))
            assert covered == list(range(N))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    D.init_from_env("gloo")
    N = 8
    lo, hi = D.shard_range(N, rank, world)
    # a per-image "chain" stand-in on CPU: each image's output depends only on
    # that image (O8), physical layout N outermost
    g = torch.Generator().manual_seed(0)
    batch = torch.randn(N, 4, 3, 3, generator=g)
    w = torch.randn(5, 4, generator=g)
    local = torch.einsum("nchw,kc->nkhw", batch[lo:hi], w).contiguous()
    full = D.gather_outputs(local, world)
    t = D.max_over_ranks(float(rank + 1), world)
    q.put((rank, full, t))
    dist.destroy_process_group()


def test_gloo_gather_and_max_world2():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = torch.Generator().manual_seed(0)
    batch = torch.randn(8, 4, 3, 3, generator=g)
    w = torch.randn(5, 4, generator=g)
    want = torch.einsum("nchw,kc->nkhw", batch, w)
    for rank, full, t in res:
        assert torch.equal(full, want)      # shards reassembled in rank order
        assert t == 2.0                     # max over ranks
