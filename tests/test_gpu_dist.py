"""Batch-sharded R18 chain on the GPU (row a10, BASELINE config 5): each rank
runs the whole chain on its shard of the global batch through the C-ABI and
one all-gather (NCCL) assembles the 512x7x7 outputs.  The gathered output is
compared image by image with the fp64 oracle (teacher-forced through every op
of the shard, then the final op's output read from the GATHERED buffer), at
world size 1 and, when two GPUs are visible, at world size 2 over NCCL."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import dist as D
from tests.helpers import BF16_TOL, norm_rel, words
from tests.test_gpu_fullsize import _check_chain_images

pytestmark = pytest.mark.gpu


def _final_vs_oracle(ch: CH.Chain, gathered: torch.Tensor, lo: int, images):
    """the last conv's oracle output for shard images, compared with the rows
    lo + n of the gathered buffer"""
    i = len(ch.ops) - 1
    op = ch.ops[i]
    assert op[0] == "conv"
    L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
    wl, w, sc, bi = ch.weights[i]
    shp = lambda t: (1,) + tuple(ch.shapes[t][1:])  # noqa: E731
    Ox = oracle.Layout(shp(src), ch.layouts[src].prims)
    Ow = oracle.Layout(wl.logical_shape, wl.prims)
    pd = dict(N=1, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride, stride_w=L.stride,
              pad_h=L.pad, pad_w=L.pad)
    for n in images:
        kw = {}
        if res is not None:
            kw = dict(res_l=oracle.Layout(shp(res), ch.layouts[res].prims), residual=words(ch.buf[res][n:n + 1]))
        ref = oracle.conv2d(pd, Ox, words(ch.buf[src][n:n + 1]), Ow, words(w), scale=sc.double().cpu().numpy(),
                            bias=bi.double().cpu().numpy(), act=1 if relu else 0, **kw)
        got = oracle.Layout(shp(dst), ch.layouts[dst].prims).read_f64(words(gathered[lo + n:lo + n + 1]))
        err = norm_rel(got, ref)
        assert err <= BF16_TOL, (n, err)


def test_sharded_r18_world1_shard32():
    """the 8-GPU shard configuration (batch 32 of 256, chain_tune r18|N32)
    at world 1: shard = whole batch, gather = identity, outputs vs oracle"""
    dev = torch.device("cuda", 0)
    holder = {}

    def run_shard(lo, hi):
        ch = CH.resnet18(hi - lo, dev)
        holder["ch"] = ch
        return ch.run()
    full = D.sharded_forward(32, 1, 0, run_shard)
    torch.cuda.synchronize()
    ch = holder["ch"]
    assert full.shape[0] == 32
    _final_vs_oracle(ch, full, 0, images=(0, 13, 31))


@pytest.mark.parametrize("N", [128, 64, 32])
def test_r18_shard_configs_every_op(N):
    """every op of the chain at the per-GPU shard batches of 2 / 4 / 8 GPUs
    (tuned chain configs), teacher-forced, images spread over the batch"""
    ch = CH.resnet18(N, torch.device("cuda", 0))
    _check_chain_images(ch, relu6=False, images=(0, N // 3, N - 1))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, N, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    D.init_from_env("nccl")
    dev = torch.device("cuda", rank)
    holder = {}

    def run_shard(lo, hi):
        ch = CH.resnet18(hi - lo, dev)
        holder["ch"] = ch
        return ch.run()
    full = D.sharded_forward(N, world, rank, run_shard)
    torch.cuda.synchronize()
    lo, hi = D.shard_range(N, rank, world)
    ok = torch.equal(full[lo:hi].view(torch.int16), holder["ch"].buf[holder["ch"].out_name].view(torch.int16))
    err = None
    try:
        _final_vs_oracle(holder["ch"], full, lo, images=(0, hi - lo - 1))
    except AssertionError as e:
        err = str(e)
    q.put((rank, ok, err))
    torch.distributed.destroy_process_group()


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs 2 visible GPUs")
def test_sharded_r18_world2_nccl():
    world, port, N = 2, _free_port(), 64
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, N, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank, ok, err in res:
        assert ok, f"rank {rank}: its gathered rows differ from its shard"
        assert err is None, err
