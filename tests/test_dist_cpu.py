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


# A two-conv chain over ALT layouts (conv 3x3 + BN + ReLU -> conv 1x1 with
# the first conv's output as residual-free input), evaluated per shard by the
# fp64 oracle (tests may call oracle/); the host logic under test is the
# product's sharded_forward: shard ranges, per-rank chain, uneven all-gather.
CHAIN_N, CHAIN_C, CHAIN_HW, CHAIN_K = 5, 8, 6, 16
LX = [("split", 1, [1, 8]), ("reorder", [0, 1, 3, 4, 2])]                 # NCHW8c
LW1 = [("split", 0, [2, 8]), ("split", 2, [1, 8]), ("reorder", [0, 2, 4, 5, 1, 3])]
LY1 = [("split", 1, [2, 8]), ("reorder", [0, 1, 3, 4, 2])]
LW2 = [("reorder", [0, 2, 3, 1])]


def _chain_inputs():
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth
    x = synth.activations("gloo_x", (CHAIN_N, CHAIN_C, CHAIN_HW, CHAIN_HW)).float().numpy()
    w1 = synth.weights("gloo_w1", (CHAIN_K, CHAIN_C, 3, 3)).float().numpy()
    w2 = synth.weights("gloo_w2", (CHAIN_K, CHAIN_K, 1, 1)).float().numpy()
    return x, w1, w2


def _oracle_chain(lo, hi):
    """images [lo, hi) through the chain, activations stored in ALT layouts
    between the ops; returns the shard's output (N outermost, fp64)."""
    import numpy as np
    import oracle
    x, w1, w2 = _chain_inputs()
    n = hi - lo
    words = lambda a: np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)  # noqa: E731
    Ox = oracle.Layout((n, CHAIN_C, CHAIN_HW, CHAIN_HW), LX)
    Ow1 = oracle.Layout(w1.shape, LW1)
    p1 = dict(N=n, C=CHAIN_C, H=CHAIN_HW, W=CHAIN_HW, K=CHAIN_K, R=3, S=3, pad_h=1, pad_w=1)
    y1 = oracle.conv2d(p1, Ox, Ox.materialize(words(x[lo:hi])), Ow1, Ow1.materialize(words(w1)), act=1)
    Oy1 = oracle.Layout(y1.shape, LY1)
    Ow2 = oracle.Layout(w2.shape, LW2)
    p2 = dict(N=n, C=CHAIN_K, H=CHAIN_HW, W=CHAIN_HW, K=CHAIN_K, R=1, S=1)
    y2 = oracle.conv2d(p2, Oy1, Oy1.materialize(words(y1)), Ow2, Ow2.materialize(words(w2)))
    return torch.from_numpy(np.ascontiguousarray(y2))


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    D.init_from_env("gloo")
    full = D.sharded_forward(CHAIN_N, world, rank, _oracle_chain)   # N = 5: uneven shards (3 + 2)
    t = D.max_over_ranks(float(rank + 1), world)
    q.put((rank, full, t))
    dist.destroy_process_group()


def test_gloo_sharded_chain_world2():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=180) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    want = _oracle_chain(0, CHAIN_N)          # the unsharded chain
    for rank, full, t in res:
        assert full.shape == want.shape
        assert torch.equal(full, want)        # shards reassembled in rank order, padding dropped
        assert t == 2.0                       # max over ranks
