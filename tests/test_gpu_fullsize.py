"""Parity at BASELINE.json's full sizes, in the launch configurations
bench.py times (tuned layouts and kernel configurations from tune_cache.jsonl
/ chain_tune.json, CUDA-graph-free eager launches of the same plans).

Images are independent (O8).  Every output element of the ResNet-50 set (all
32 images of every layer, and the batch-1 plans), of the MobileNet-V2 chain
(all 16 images of every op) and of the BERT GEMMs (all 8192 rows) is
compared with the fp64 oracle, and for ResNet-18 at batch 256 sixteen images
spread over every wave of the persistent tile schedule.  Two bars per output
(tests/helpers.py): the normwise 2e-2 per image, and the per-element
envelope |y - ref| <= 2^-7 (|ref| + |scale| sum|x w| + |bias| + |res|), which
a single corrupted row or stale tile fails.  Chains are teacher-forced (each
op's oracle reads the GPU's own input of that op)."""
import numpy as np
import pytest
import torch

import bench
import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets
from tests.helpers import BF16_TOL, abs_conv_ref, assert_elementwise, norm_rel, words

pytestmark = pytest.mark.gpu


def _image(t: torch.Tensor, n: int) -> np.ndarray:
    """words of image n of a physical buffer whose outermost dim is N"""
    return words(t[n:n + 1])


def _check_layer_set(S):
    """every image of every layer of a bench.LayerSet against O3 + O6"""
    worst = 0.0
    for l in S.layers:
        L = l["L"]
        N = S.N
        Ho, Wo = L.out_hw()
        Ox = oracle.Layout((N, L.C, L.H, L.W), l["lx"].prims)
        Ow = oracle.Layout((L.K, L.C, L.R, L.S), l["lw"].prims)
        Oy = oracle.Layout((N, L.K, Ho, Wo), l["ly"].prims)
        xl, wl = Ox.read_f64(words(l["x"])), Ow.read_f64(words(l["w"]))
        sc, bi = l["sc"].double().cpu().numpy(), l["bi"].double().cpu().numpy()
        pd = dict(N=N, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride, stride_w=L.stride,
                  pad_h=L.pad, pad_w=L.pad)
        ref = oracle.conv2d_f64(pd, xl, wl, sc, bi, None, 1)
        absref = abs_conv_ref(pd, xl, wl, sc, bi)
        yw = words(l["y"])
        assert Oy.check_consistent(yw) == 0, L.name   # pad zeros / unfold copies
        got = Oy.read_f64(yw)
        for n in range(N):
            err = norm_rel(got[n], ref[n])
            worst = max(worst, err)
            assert err <= BF16_TOL, (L.name, n, err)
        assert_elementwise(got, ref, absref, L.name)
    assert worst > 0.0  # bf16 outputs: an exact match would mean the check compared nothing
    return worst


def test_r50_layer_set_b32_bench_config():
    """BASELINE config 2 as bench.py runs it: 23 layers at batch 32 with the
    tuned plans; all 32 images of every layer against the oracle (O3+O6)."""
    dev = torch.device("cuda", 0)
    S = bench.LayerSet(32, dev)
    S.step()
    torch.cuda.synchronize()
    _check_layer_set(S)
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


def test_r50_layer_set_b1_tuned_plans():
    """BASELINE config 2 at batch 1 (the tune cache's N1 plans)"""
    S = bench.LayerSet(1, torch.device("cuda", 0))
    S.step()
    torch.cuda.synchronize()
    _check_layer_set(S)


def _check_chain_images(ch: CH.Chain, relu6: bool, images):
    ch.run()
    torch.cuda.synchronize()
    images = list(images)
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
                xl, wlg = Ox.read_f64(_image(ch.buf[src], n)), Ow.read_f64(words(w))
                rl = None
                if res is not None:
                    rl = oracle.Layout(shp(res), ch.layouts[res].prims).read_f64(_image(ch.buf[res], n))
                act = (2 if relu6 else 1) if relu else 0
                scd, bid = sc.double().cpu().numpy(), bi.double().cpu().numpy()
                ref = oracle.conv2d_f64(pd, xl, wlg, scd, bid, rl, act)
                Oy = oracle.Layout(shp(dst), ch.layouts[dst].prims)
                yw = _image(ch.buf[dst], n)
                assert Oy.check_consistent(yw) == 0, (L.name, n)
                got = Oy.read_f64(yw)
                err = norm_rel(got, ref)
                assert err <= BF16_TOL, (L.name, n, err)
                assert_elementwise(got, ref, abs_conv_ref(pd, xl, wlg, scd, bid, rl), f"{L.name} image {n}")
            else:
                _, k, s, p, src, dst = op
                Ox = oracle.Layout((1,) + tuple(ch.shapes[src][1:]), ch.layouts[src].prims)
                ref = oracle.pool2d_f64(Ox.read_f64(_image(ch.buf[src], n)), k, k, s, p, "max")
                got = oracle.Layout((1,) + tuple(ch.shapes[dst][1:]), ch.layouts[dst].prims).read_f64(
                    _image(ch.buf[dst], n))
                assert np.array_equal(got, ref)


def test_resnet18_chain_b256_bench_config():
    """BASELINE config 5 at its 1-GPU shard (batch 256, tuned chain configs):
    16 images spread over the batch — every wave of the persistent tile
    schedule of the large early layers — through every op, teacher-forced."""
    ch = CH.resnet18(256, torch.device("cuda", 0))
    assert ch.cfgs_loaded or not ch.cfgs
    images = sorted(set([0, 255] + [int(v) for v in np.linspace(1, 254, 14)]))
    assert len(images) == 16
    _check_chain_images(ch, relu6=False, images=images)


def test_mobilenet_v2_chain_b16_bench_config():
    """BASELINE config 4 (batch 16, tuned chain configs): all 16 images"""
    ch = CH.mobilenet_v2(16, torch.device("cuda", 0))
    _check_chain_images(ch, relu6=True, images=range(16))


@pytest.mark.parametrize("gemm", nets.BERT_GEMMS, ids=[g[0] for g in nets.BERT_GEMMS])
def test_bert_gemm_m8192_bench_config(gemm):
    """BASELINE config 3 as bench.py runs it (M = 8192, tiled layouts, the
    tuned kernel configuration): all 8192 rows against the oracle (O5),
    normwise per 512-row block and the per-element envelope."""
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
    Al, Bl = Oa.read_f64(aw), Ob.read_f64(bw)
    ref = oracle.gemm_f64(Al, Bl)
    absref = oracle.gemm_f64(np.abs(Al), np.abs(Bl))
    for m0 in range(0, M, 512):
        err = norm_rel(got[m0:m0 + 512], ref[m0:m0 + 512])
        assert err <= BF16_TOL, (name, m0, err)
    assert_elementwise(got, ref, absref, name)
