"""Parity at BASELINE.json's full sizes, in the launch configurations
bench.py times (tuned layouts and kernel configurations from tune_cache.jsonl
/ chain_tune.json, CUDA-graph-free eager launches of the same plans).

Images are independent (O8), so whole output images are checked exactly
against the fp64 oracle: the first and the last image of every batch
(SURVEY §8d "deterministic subset of images").  Chains are teacher-forced
(each op's oracle reads the GPU's own input of that op).  BERT GEMMs check
row blocks at both ends of M = 8192."""
import numpy as np
import pytest
import torch

import bench
import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets
from tests.helpers import BF16_TOL, norm_rel, words

pytestmark = pytest.mark.gpu


def _image(t: torch.Tensor, n: int) -> np.ndarray:
    """words of image n of a physical buffer whose outermost dim is N"""
    return words(t[n:n + 1])


def test_r50_layer_set_b32_bench_config():
    """BASELINE config 2 as bench.py runs it: 23 layers at batch 32 with the
    tuned plans; images 0 and 31 of every layer against the oracle (O3+O6)."""
    dev = torch.device("cuda", 0)
    S = bench.LayerSet(32, dev)
    S.step()
    torch.cuda.synchronize()
    worst = 0.0
    for l in S.layers:
        L = l["L"]
        Ho, Wo = L.out_hw()
        Ox = oracle.Layout((1, L.C, L.H, L.W), l["lx"].prims)
        Ow = oracle.Layout((L.K, L.C, L.R, L.S), l["lw"].prims)
        Oy = oracle.Layout((1, L.K, Ho, Wo), l["ly"].prims)
        wph = words(l["w"])
        pd = dict(N=1, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride, stride_w=L.stride,
                  pad_h=L.pad, pad_w=L.pad)
        for n in (0, 31):
            ref = oracle.conv2d(pd, Ox, _image(l["x"], n), Ow, wph, scale=l["sc"].double().cpu().numpy(),
                                bias=l["bi"].double().cpu().numpy(), act=1)
            got = Oy.read_f64(_image(l["y"], n))
            err = norm_rel(got, ref)
            worst = max(worst, err)
            assert err <= BF16_TOL, (L.name, n, err)
    assert worst > 0.0  # bf16 outputs: an exact match would mean the check compared nothing
    # the e2e path (copies on their own streams, events ordering every buffer
    # reuse across steps) delivers the same outputs to the host
    for l in S.layers:
        l["y"].zero_()
    for _ in range(2):
        S.step_e2e_overlap()
    torch.cuda.synchronize()
    S.step()
    torch.cuda.synchronize()
    for l in S.layers:
        assert np.array_equal(words(l["y_host"]), words(l["y"])), l["L"].name


def _check_chain_images(ch: CH.Chain, relu6: bool, images):
    ch.run()
    torch.cuda.synchronize()
    for i, op in enumerate(ch.ops):
        for n in images:
            if op[0] == "conv":
                L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
                wl, w, sc, bi = ch.weights[i]
                shp = lambda t: (1,) + tuple(ch.shapes[t][1:])  # noqa: E731
                Ox = oracle.Layout(shp(src), ch.layouts[src].prims)
                Ow = oracle.Layout(wl.logical_shape, wl.prims)
                pd = dict(N=1, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride,
                          stride_w=L.stride, pad_h=L.pad, pad_w=L.pad, groups=L.groups)
                kw = {}
                if res is not None:
                    kw = dict(res_l=oracle.Layout(shp(res), ch.layouts[res].prims),
                              residual=_image(ch.buf[res], n))
                act = (2 if relu6 else 1) if relu else 0
                ref = oracle.conv2d(pd, Ox, _image(ch.buf[src], n), Ow, words(w),
                                    scale=sc.double().cpu().numpy(), bias=bi.double().cpu().numpy(), act=act,
                                    **kw)
                got = oracle.Layout(shp(dst), ch.layouts[dst].prims).read_f64(_image(ch.buf[dst], n))
                err = norm_rel(got, ref)
                assert err <= BF16_TOL, (L.name, n, err)
            else:
                _, k, s, p, src, dst = op
                Ox = oracle.Layout((1,) + tuple(ch.shapes[src][1:]), ch.layouts[src].prims)
                ref = oracle.pool2d_f64(Ox.read_f64(_image(ch.buf[src], n)), k, k, s, p, "max")
                got = oracle.Layout((1,) + tuple(ch.shapes[dst][1:]), ch.layouts[dst].prims).read_f64(
                    _image(ch.buf[dst], n))
                assert np.array_equal(got, ref)


def test_resnet18_chain_b256_bench_config():
    """BASELINE config 5 at its 1-GPU shard (batch 256, tuned chain configs):
    images 0 and 255 through every op, teacher-forced."""
    ch = CH.resnet18(256, torch.device("cuda", 0))
    assert ch.cfgs_loaded or not ch.cfgs
    _check_chain_images(ch, relu6=False, images=(0, 255))


def test_mobilenet_v2_chain_b16_bench_config():
    """BASELINE config 4 (batch 16, tuned chain configs): images 0 and 15."""
    ch = CH.mobilenet_v2(16, torch.device("cuda", 0))
    _check_chain_images(ch, relu6=True, images=(0, 15))


@pytest.mark.parametrize("gemm", nets.BERT_GEMMS, ids=[g[0] for g in nets.BERT_GEMMS])
def test_bert_gemm_m8192_bench_config(gemm):
    """BASELINE config 3 as bench.py runs it (M = 8192, tiled layouts, the
    tuned kernel configuration): rows [0, 256) and [M - 256, M) against the
    oracle (O5)."""
    name, K, N = gemm
    M = 8192
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth
    A = synth.activations("fsA" + name, (M, K)).to(torch.bfloat16)
    B = synth.weights("fsB" + name, (K, N)).to(torch.bfloat16)
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import tunecache
    cfg = dict(tunecache.lookup_gemm(M, N, K) or {"path": 1, "block_n": 256})
    nt = cfg.pop("b_nt", 256)
    ap, bp, cp = LY.gemm_a_tiled(M, K, 128, 64), LY.gemm_b_tiled_nk(K, N, nt, 64), LY.gemm_c_tiled(M, N, 128, 64)
    La, Lb, Lc = alt.Layout((M, K), ap), alt.Layout((K, N), bp), alt.Layout((M, N), cp)
    Oa, Ob, Oc = oracle.Layout((M, K), ap), oracle.Layout((K, N), bp), oracle.Layout((M, N), cp)
    aw = Oa.materialize(words(A).reshape(M, K))
    bw = Ob.materialize(words(B).reshape(K, N))
    a = torch.from_numpy(aw.view(np.int16)).view(torch.bfloat16).cuda()
    b = torch.from_numpy(bw.view(np.int16)).view(torch.bfloat16).cuda()
    c = Lc.empty(torch.bfloat16)
    alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg=cfg)
    torch.cuda.synchronize()
    got = Oc.read_f64(words(c))
    for m0, m1 in ((0, 256), (M - 256, M)):
        ref = oracle.gemm(Oa, aw, Ob, bw, rows=(m0, m1))[m0:m1]
        err = norm_rel(got[m0:m1], ref)
        assert err <= BF16_TOL, (name, m0, err)
