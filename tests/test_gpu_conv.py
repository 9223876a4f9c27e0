"""GPU parity of alt_conv2d / alt_matmul against the fp64 oracle, every path
(tensor-core tcgen05, SIMT generic, depthwise), many layouts, fused
epilogue, pad-zero / unfold-copy consistency of outputs, invariants I2
(layout independence) and I3 (pad/unfold input == direct conv)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth
from tests.helpers import assert_parity, make_operand, read_output, words

pytestmark = pytest.mark.gpu


def run_conv(name, N, C, H, W, K, R, S, V, pad, xp, wp, yp, dtype, groups=1, epi=False,
             res_p=None, act=0, cfg=None, expect_path=None, dil=1):
    x = synth.activations(name + "x", (N, C, H, W))
    w = synth.weights(name + "w", (K, C // groups, R, S))
    Ho, Wo = (H + 2 * pad - dil * (R - 1) - 1) // V + 1, (W + 2 * pad - dil * (S - 1) - 1) // V + 1
    Xo, xph, xd = make_operand(name, xp, x, dtype)
    Wo_, wph, wd = make_operand(name, wp, w, dtype)
    p = alt.conv_params(N, C, H, W, K, R, S, V, pad, groups, dilation=dil)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((N, K, Ho, Wo), yp)
    y = torch.full(Ly.phys_shape, 3.0, dtype=dtype, device="cuda")  # poison
    kw = {}
    ref_kw = {}
    if epi:
        sc, bi = synth.bn_scale(name + "s", K), synth.bn_bias(name + "b", K)
        kw.update(scale=sc.cuda(), bias=bi.cuda())
        ref_kw.update(scale=sc.double().numpy(), bias=bi.double().numpy())
    if res_p is not None:
        r = synth.activations(name + "r", (N, K, Ho, Wo))
        Ro, rph, rd = make_operand(name + "r", res_p, r, dtype)
        kw.update(residual=rd, residual_l=alt.Layout((N, K, Ho, Wo), res_p))
        ref_kw.update(res_l=Ro, residual=rph)
    alt.conv2d(p, Lx, xd, Lw, wd, Ly, y, act=act, cfg=cfg, **kw)
    plan = alt.last_plan()
    torch.cuda.synchronize()
    if expect_path is not None:
        assert plan["path"] == expect_path, plan
    pd = dict(N=N, C=C, H=H, W=W, K=K, R=R, S=S, stride_h=V, stride_w=V, pad_h=pad, pad_w=pad,
              groups=groups, dil_h=dil, dil_w=dil)
    ref = oracle.conv2d(pd, Xo, xph, Wo_, wph, act=act, **ref_kw)
    got = read_output(oracle.Layout((N, K, Ho, Wo), yp), y, dtype)
    return assert_parity(got, ref, dtype), plan


# ---------------------------------------------------------------- config 1 --
D1 = dict(N=1, C=16, H=14, W=14, K=32, R=3, S=3, V=1, pad=1)
D1_LAYOUTS = [
    ("NCHW", [], [], []),
    ("NCHW4c/KCRS4k4c", LY.nchwxc(16, 4), LY.kcrs_yk_xc(32, 16, 4, 4), LY.nchwxc(32, 4)),
    ("NHWC/KRSC", LY.nhwc(), [("reorder", [0, 2, 3, 1])], LY.nhwc()),
    ("NCHW8c/KCRS16k8c", LY.nchwxc(16, 8), LY.kcrs_yk_xc(32, 16, 16, 8), LY.nchwxc(32, 16)),
    ("tiled unfold in/out", LY.conv_input_tiled(16, 8, 14, 14, 3, 3, 7, 7, 1, 1),
     LY.kcrs_paper(32, 16, 16, 8), LY.conv_output_tiled(32, 16, 14, 14, 7, 7)),
    ("padded NCHW16c", LY.nchwxc(16, 16, pad_hw=1), LY.kcrs_yk_xc(32, 16, 32, 16), LY.nchwxc(32, 32)),
]


@pytest.mark.parametrize("lay", D1_LAYOUTS, ids=[l[0] for l in D1_LAYOUTS])
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("path", [alt.PATH_AUTO, alt.PATH_SIMT])
def test_config1_conv_layouts(lay, dtype, path):
    _, xp, wp, yp = lay
    run_conv("d1" + lay[0], **D1, xp=xp, wp=wp, yp=yp, dtype=dtype, cfg={"path": path})


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("act", [0, 1, 2])
def test_epilogue_scale_bias_residual_act(dtype, act):
    run_conv("epi", 2, 16, 9, 11, 24, 3, 3, 1, 1, LY.nchwxc(16, 8), LY.kcrs_yk_xc(24, 16, 8, 8),
             LY.nchwxc(24, 8), dtype, epi=True, res_p=LY.nhwc(), act=act)


def test_output_pad_and_unfold_copies_written():
    """The epilogue writes the consumer's tiled + padded input layout
    directly (propagation, Fig. 5b): zeros in pads, all unfold copies."""
    yp = LY.conv_input_tiled(16, 8, 14, 14, 3, 3, 7, 7, 1, 1)
    run_conv("propout", 2, 16, 14, 14, 16, 3, 3, 1, 1, LY.nchwxc(16, 16), LY.kcrs_yk_xc(16, 16, 16, 16),
             yp, torch.bfloat16, epi=True, act=1)


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
def test_depthwise_and_grouped(dtype):
    run_conv("dw", 2, 32, 14, 14, 32, 3, 3, 1, 1, LY.nchwxc(32, 8), [], LY.nchwxc(32, 8), dtype,
             groups=32, epi=True, act=2)
    run_conv("dw2", 2, 32, 15, 15, 32, 3, 3, 2, 1, LY.nchwxc(32, 16), [], LY.nchwxc(32, 16), dtype,
             groups=32)
    run_conv("grp", 2, 16, 9, 9, 32, 3, 3, 1, 1, [], [], [], dtype, groups=4)


DW_CASES = [  # (name, N, C, H, W, R, V, pad, x/y layout, residual layout)
    ("dw_rsk_c64", 2, 64, 14, 13, 3, 1, 1, LY.nchwxc(64, 64), LY.nchwxc(64, 64)),
    ("dw_rsk_s2", 3, 48, 15, 15, 3, 2, 1, LY.nchwxc(48, 16), None),
    ("dw_rsk_5x5", 1, 32, 12, 9, 5, 1, 2, LY.nchwxc(32, 8), LY.nchwxc(32, 32)),
    ("dw_rsk_1x1", 2, 24, 7, 7, 1, 1, 0, LY.nchwxc(24, 8), None),
]


@pytest.mark.parametrize("case", DW_CASES, ids=[c[0] for c in DW_CASES])
def test_depthwise_vector_weights(case):
    """Depthwise fast path: weights stored R S K (8 consecutive k contiguous
    per tap), 16-byte residual vectors, every channel-run ordering."""
    name, N, C, H, W, R, V, pad, xp, rp = case
    run_conv(name, N, C, H, W, C, R, R, V, pad, xp, [("reorder", [1, 2, 3, 0])], xp, torch.bfloat16,
             groups=C, epi=True, act=2, res_p=rp, expect_path=alt.PATH_DW)


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
def test_layout_independence_I2(dtype):
    outs = []
    for i, (_, xp, wp, yp) in enumerate(D1_LAYOUTS):
        outs.append(run_conv("i2", **D1, xp=xp, wp=wp, yp=yp, dtype=dtype)[0])
    assert max(outs) <= (1e-5 if dtype == torch.float32 else 2e-2)


def test_pad_unfold_input_equals_direct_I3():
    # same data, semantic padding vs materialised pad + unfold input layouts
    for xp in ([], LY.nchwxc(16, 8, pad_hw=1), LY.conv_input_tiled(16, 8, 14, 14, 3, 3, 7, 7, 1, 1)):
        run_conv("i3", **D1, xp=xp, wp=LY.kcrs_yk_xc(32, 16, 16, 8), yp=LY.nchwxc(32, 16),
                 dtype=torch.float32)


# -------------------------------------------------------------------- GEMM --
def run_gemm(name, M, N, K, ap, bp, cp, dtype, epi=False, cfg=None, expect_path=None):
    A = synth.activations(name + "A", (M, K))
    B = synth.weights(name + "B", (K, N))
    Ao, aph, ad = make_operand(name + "A", ap, A, dtype)
    Bo, bph, bd = make_operand(name + "B", bp, B, dtype)
    La, Lb, Lc = alt.Layout((M, K), ap), alt.Layout((K, N), bp), alt.Layout((M, N), cp)
    c = torch.full(Lc.phys_shape, 5.0, dtype=dtype, device="cuda")
    kw, ref_kw = {}, {}
    if epi:
        bi = synth.bn_bias(name + "b", N)
        kw.update(bias=bi.cuda(), act=1)
        ref_kw.update(bias=bi.double().numpy(), act=1)
    alt.matmul(M, N, K, La, ad, Lb, bd, Lc, c, cfg=cfg, **kw)
    plan = alt.last_plan()
    torch.cuda.synchronize()
    if expect_path is not None:
        assert plan["path"] == expect_path, plan
    ref = oracle.gemm(Ao, aph, Bo, bph, **ref_kw)
    got = read_output(oracle.Layout((M, N), cp), c, dtype)
    return assert_parity(got, ref, dtype), plan


GEMM_LAYOUTS = [
    ("MK/KN/MN", [], [], []),
    ("MK/NK(col)/MN", [], LY.transpose2(), []),
    ("tiled template", LY.gemm_a_tiled(256, 192, 64, 64), LY.gemm_b_tiled_kn(192, 128, 64, 64),
     LY.gemm_c_tiled(256, 128, 64, 64)),
    ("NKn", [("split", 0, [16, 16]), ("reorder", [0, 2, 1])], LY.gemm_nkn_b(192, 128), []),
]


@pytest.mark.parametrize("lay", GEMM_LAYOUTS, ids=[l[0] for l in GEMM_LAYOUTS])
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("path", [alt.PATH_AUTO, alt.PATH_SIMT])
def test_gemm_layouts(lay, dtype, path):
    _, ap, bp, cp = lay
    run_gemm("g" + lay[0], 256, 128, 192, ap, bp, cp, dtype, epi=True, cfg={"path": path})


# ------------------------------------------------------ tensor-core path --
TC_CASES = [
    # name, (N, C, H, W, K, R, S, V, pad), x prims, w prims, y prims
    ("NCHW64c 3x3", (2, 64, 14, 14, 128, 3, 3, 1, 1), LY.nchwxc(64, 64), LY.kcrs_yk_xc(128, 64, 128, 64),
     LY.nchwxc(128, 64)),
    ("NHWC 3x3 C128", (2, 128, 10, 12, 64, 3, 3, 1, 1), LY.nhwc(), [("reorder", [0, 2, 3, 1])], LY.nhwc()),
    ("NCHW16c/KCRS16k16c", (2, 32, 9, 9, 64, 3, 3, 1, 1), LY.nchwxc(32, 16), LY.kcrs_yk_xc(64, 32, 16, 16),
     LY.nchwxc(64, 16)),
    ("NCHW8c/KCRS32k8c", (2, 16, 11, 7, 64, 3, 3, 1, 1), LY.nchwxc(16, 8), LY.kcrs_yk_xc(64, 16, 32, 8),
     LY.nchwxc(64, 8)),
    ("NCHW32c stride2", (4, 64, 15, 15, 64, 3, 3, 2, 1), LY.nchwxc(64, 32), LY.kcrs_yk_xc(64, 64, 64, 32),
     LY.nchwxc(64, 32)),
    ("1x1 stride2", (4, 128, 14, 14, 256, 1, 1, 2, 0), LY.nchwxc(128, 64), LY.kcrs_yk_xc(256, 128, 64, 64),
     LY.nchwxc(256, 64)),
    ("conv1 C3->8 7x7 s2", (2, 3, 32, 32, 64, 7, 7, 2, 3), LY.nchwxc(3, 8, pad_c=5),
     LY.kcrs_yk_xc(64, 3, 64, 8, pad_c=5), LY.nchwxc(64, 64)),
    ("padded input", (2, 64, 14, 14, 64, 3, 3, 1, 1), LY.nchwxc(64, 64, pad_hw=1),
     LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64)),
    ("unfold tiled input", (2, 64, 14, 14, 64, 3, 3, 1, 1),
     LY.conv_input_tiled(64, 64, 14, 14, 3, 3, 8, 8, 1, 1), LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64)),
    ("unfold tiled input s2 it16", (2, 32, 30, 30, 64, 3, 3, 2, 1),
     LY.conv_input_tiled(32, 16, 30, 30, 3, 3, 8, 8, 2, 1), LY.kcrs_yk_xc(64, 32, 64, 16), LY.nchwxc(64, 32)),
    ("unfold out tiled", (2, 64, 14, 14, 128, 3, 3, 1, 1), LY.nchwxc(64, 64), LY.kcrs_yk_xc(128, 64, 128, 64),
     LY.conv_output_tiled(128, 16, 14, 14, 7, 7)),
    # window-folded input (unfold B = E, step = V; reading A23): conv1-like
    ("wfold conv1 C3 7x7 s2", (2, 3, 38, 38, 64, 7, 7, 2, 3), LY.conv_input_wfold(3, 7, 2, 3),
     LY.kcrs_wfold(64, 3, 7), LY.nchwxc(64, 64)),
    ("wfold C3 3x3 s2 K32", (3, 3, 30, 26, 32, 3, 3, 2, 1), LY.conv_input_wfold(3, 3, 2, 1),
     LY.kcrs_wfold(32, 3, 3), LY.nchwxc(32, 32)),
    ("wfold C16 3x3 s1", (2, 16, 12, 20, 64, 3, 3, 1, 1), LY.conv_input_wfold(16, 3, 1, 1),
     LY.kcrs_wfold(64, 16, 3), LY.nhwc()),
]


@pytest.mark.parametrize("case", TC_CASES, ids=[c[0] for c in TC_CASES])
def test_tc_conv(case):
    name, (N, C, H, W, K, R, S, V, pad), xp, wp, yp = case
    run_conv("tc" + name, N, C, H, W, K, R, S, V, pad, xp, wp, yp, torch.bfloat16, epi=True, act=1,
             cfg={"path": alt.PATH_TC}, expect_path=alt.PATH_TC)


def test_tc_unavailable_layout_falls_back_to_simt():
    """ht = 7 unfold tiles cannot hold a 128-row tensor-core tile: AUTO runs
    the generic path (still exact), TC reports ALT_E_UNSUPPORTED."""
    xp = LY.conv_input_tiled(64, 64, 14, 14, 3, 3, 7, 7, 1, 1)
    _, plan = run_conv("fallback", 2, 64, 14, 14, 64, 3, 3, 1, 1, xp, LY.kcrs_yk_xc(64, 64, 64, 64),
                       LY.nchwxc(64, 64), torch.bfloat16)
    assert plan["path"] == alt.PATH_SIMT
    with pytest.raises(alt.AltError) as e:
        run_conv("fallback", 2, 64, 14, 14, 64, 3, 3, 1, 1, xp, LY.kcrs_yk_xc(64, 64, 64, 64),
                 LY.nchwxc(64, 64), torch.bfloat16, cfg={"path": alt.PATH_TC})
    assert e.value.code == alt._alt.ALT_E_UNSUPPORTED


@pytest.mark.parametrize("bn", [64, 128, 256])
def test_tc_conv_block_n_and_residual(bn):
    run_conv("tcbn", 2, 64, 16, 16, 256, 3, 3, 1, 1, LY.nchwxc(64, 64), LY.kcrs_yk_xc(256, 64, 256, 64),
             LY.nchwxc(256, 64), torch.bfloat16, epi=True, res_p=LY.nchwxc(256, 64), act=1,
             cfg={"path": alt.PATH_TC, "block_n": bn}, expect_path=alt.PATH_TC)


TC_GEMM = [
    ("MK/NK", [], LY.transpose2(), []),
    ("tiled K-major", LY.gemm_a_tiled(384, 256, 128, 64), LY.gemm_b_tiled_nk(256, 192, 64, 64),
     LY.gemm_c_tiled(384, 192, 128, 64)),
    ("tiled mt=64 kt=32", LY.gemm_a_tiled(384, 256, 64, 32), LY.gemm_b_tiled_nk(256, 192, 64, 32), []),
]


@pytest.mark.parametrize("case", TC_GEMM, ids=[c[0] for c in TC_GEMM])
def test_tc_gemm(case):
    name, ap, bp, cp = case
    run_gemm("tcg" + name, 384, 192, 256, ap, bp, cp, torch.bfloat16, epi=True, cfg={"path": alt.PATH_TC},
             expect_path=alt.PATH_TC)


# ------------------------------------------------------------- split-K --
@pytest.mark.parametrize("sk,bn,pair", [(2, 256, 1), (3, 128, 1), (5, 64, 2), (0, 256, 0)])
def test_tc_split_k(sk, bn, pair):
    """split-K (alt_kernel_cfg.split_k; 0 = auto = none): partial tiles summed in split order by the last CTA, fused
    epilogue with residual, parity with the oracle."""
    cfg = {"path": alt.PATH_TC, "split_k": sk, "block_n": bn, "cta_pair": pair}
    xp, wp, yp = LY.nchwxc(256, 64), LY.kcrs_yk_xc(512, 256, 256, 64), LY.nchwxc(512, 64)
    _, plan = run_conv("tcsk", 2, 256, 7, 7, 512, 3, 3, 1, 1, xp, wp, yp, torch.bfloat16, epi=True,
                       res_p=LY.nchwxc(512, 64), act=1, cfg=cfg, expect_path=alt.PATH_TC)
    assert plan["split_k"] == (sk or 1)  # auto: no split


def test_tc_split_k_deterministic():
    """the reduction order is fixed: repeated launches agree bit for bit"""
    p = alt.conv_params(2, 256, 7, 7, 512, 3, 3, 1, 1)
    x = synth.activations("skdx", (2, 256, 7, 7))
    w = synth.weights("skdw", (512, 256, 3, 3))
    xp, wp, yp = LY.nchwxc(256, 64), LY.kcrs_yk_xc(512, 256, 256, 64), LY.nchwxc(512, 64)
    _, _, xd = make_operand("skdx", xp, x, torch.bfloat16)
    _, _, wd = make_operand("skdw", wp, w, torch.bfloat16)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((2, 512, 7, 7), yp)
    outs = []
    for _ in range(4):
        y = torch.zeros(Ly.phys_shape, dtype=torch.bfloat16, device="cuda")
        alt.conv2d(p, Lx, xd, Lw, wd, Ly, y, cfg={"path": alt.PATH_TC, "split_k": 7})
        outs.append(y)
    torch.cuda.synchronize()
    for y in outs[1:]:
        assert np.array_equal(words(y), words(outs[0]))


def test_tc_gemm_split_k():
    _, plan = run_gemm("gsk", 200, 256, 2048, [], LY.transpose2(), [], torch.bfloat16, epi=True,
                       cfg={"path": alt.PATH_TC, "split_k": 4}, expect_path=alt.PATH_TC)
    assert plan["split_k"] == 4


# ------------------------------------------------------ cluster split-K --
@pytest.mark.parametrize("sk,bn,shape", [(2, 256, (2, 256, 7, 7, 512)), (4, 128, (2, 256, 7, 7, 512)),
                                         (4, 256, (3, 128, 9, 11, 256)), (2, 128, (1, 64, 14, 14, 128))])
def test_tc_split_cluster(sk, bn, shape):
    """cluster split-K (alt_kernel_cfg.split_cluster): the split ranges of a tile run as one thread-block
    cluster and are summed through distributed shared memory; fused BN + ReLU, ragged M tiles."""
    N, C, H, W, K = shape
    cfg = {"path": alt.PATH_TC, "split_k": sk, "block_n": bn, "cta_pair": 2, "split_cluster": 1}
    xp, wp, yp = LY.nchwxc(C, 64), LY.kcrs_yk_xc(K, C, min(K, 256), 64), LY.nchwxc(K, 64)
    _, plan = run_conv("tcsc%d%d" % (sk, bn), N, C, H, W, K, 3, 3, 1, 1, xp, wp, yp, torch.bfloat16, epi=True,
                       act=1, cfg=cfg, expect_path=alt.PATH_TC)
    assert plan["split_k"] == sk and plan["split_cluster"] == 1


def test_tc_split_cluster_deterministic_and_unsupported():
    p = alt.conv_params(2, 256, 7, 7, 512, 3, 3, 1, 1)
    x = synth.activations("scdx", (2, 256, 7, 7))
    w = synth.weights("scdw", (512, 256, 3, 3))
    xp, wp, yp = LY.nchwxc(256, 64), LY.kcrs_yk_xc(512, 256, 256, 64), LY.nchwxc(512, 64)
    _, _, xd = make_operand("scdx", xp, x, torch.bfloat16)
    _, _, wd = make_operand("scdw", wp, w, torch.bfloat16)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((2, 512, 7, 7), yp)
    cfg = {"path": alt.PATH_TC, "split_k": 4, "block_n": 256, "cta_pair": 2, "split_cluster": 1}
    outs = []
    for _ in range(3):
        y = torch.zeros(Ly.phys_shape, dtype=torch.bfloat16, device="cuda")
        alt.conv2d(p, Lx, xd, Lw, wd, Ly, y, cfg=cfg)
        outs.append(y)
    torch.cuda.synchronize()
    for y in outs[1:]:
        assert np.array_equal(words(y), words(outs[0]))
    # a residual is not served by the cluster form: the call fails loudly
    with pytest.raises(alt.AltError) as e:
        alt.conv2d(p, Lx, xd, Lw, wd, Ly, outs[0], residual=outs[1], residual_l=Ly, cfg=cfg)
    assert e.value.code == alt._alt.ALT_E_UNSUPPORTED


# ------------------------------------------- TMA-store staging reuse --
@pytest.mark.parametrize("C,K,R", [(16, 32, 3), (16, 64, 1), (3, 32, 3)])
def test_tc_many_short_tiles_tma_store(C, K, R):
    """Regression: BLOCK_N 64 tiles are one epilogue chunk each; with a short
    mainloop (few input channels) a CTA stores tile after tile, and the
    staging buffers must alternate across tiles (the previous tile's TMA store
    may still be reading).  Batch 16 at 112x112 = 784+ tiles per launch; the
    first images are the first tile of every CTA."""
    N, H = 16, 112
    x = synth.activations("ms%d%d" % (C, K), (N, C, H, H))
    w = synth.weights("msw%d%d" % (C, K), (K, C, R, R))
    if C % 8:
        xp, wp = LY.conv_input_wfold(C, R, 1, R // 2), LY.kcrs_wfold(K, C, R)
    else:
        xp, wp = LY.nchwxc(C, C), LY.kcrs_yk_xc(K, C, K, C)
    yp = LY.nchwxc(K, 32)
    Ox, _, xd = make_operand("msx", xp, x, torch.bfloat16)
    Ow, wph, wd = make_operand("msw", wp, w, torch.bfloat16)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((N, K, H, H), yp)
    y = torch.full(Ly.phys_shape, 3.0, dtype=torch.bfloat16, device="cuda")
    alt.conv2d(alt.conv_params(N, C, H, H, K, R, R, 1, R // 2), Lx, xd, Lw, wd, Ly, y,
               cfg={"path": alt.PATH_TC, "block_n": 64})
    torch.cuda.synchronize()
    assert alt.last_plan()["path"] == alt.PATH_TC
    pd = dict(N=1, C=C, H=H, W=H, K=K, R=R, S=R, stride_h=1, stride_w=1, pad_h=R // 2, pad_w=R // 2)
    Ox1, Oy1 = oracle.Layout((1, C, H, H), xp), oracle.Layout((1, K, H, H), yp)
    for n in (0, 1, N - 1):
        ref = oracle.conv2d(pd, Ox1, words(xd[n:n + 1]), Ow, wph)
        assert_parity(Oy1.read_f64(words(y[n:n + 1])), ref, torch.bfloat16)


@pytest.mark.parametrize("M,N,K", [(1024, 768, 256), (300, 384, 136)])
def test_tc_gemm_block_n_192(M, N, K):
    """BLOCK_N 192 (CTA pair, 96 B rows per CTA) on B tiled N/192 K/64"""
    _, plan = run_gemm("g192_%d" % N, M, N, K, [], LY.gemm_b_tiled_nk(K, N, 192, 8), [], torch.bfloat16, epi=True,
                       cfg={"path": alt.PATH_TC, "block_n": 192}, expect_path=alt.PATH_TC)
    assert plan["block_n"] == 192 and plan["cta_pair"] == 1


@pytest.mark.parametrize("M,N,K", [(1024, 768, 256), (300, 384, 136), (8192, 768, 768)])
def test_tc_gemm_block_n_192_single_cta(M, N, K):
    """BLOCK_N 192 on one CTA (M = 128 tiles: 4 N tiles of a 768-wide GEMM
    fill the persistent grid in 1.73 waves where 256-wide tiles need 1.3)"""
    _, plan = run_gemm("g192s_%d" % N, M, N, K, [], LY.gemm_b_tiled_nk(K, N, 192, 8), [], torch.bfloat16, epi=True,
                       cfg={"path": alt.PATH_TC, "block_n": 192, "cta_pair": 2}, expect_path=alt.PATH_TC)
    assert plan["block_n"] == 192 and plan["cta_pair"] == 2


def test_tc_conv_block_n_192_single_cta():
    """BLOCK_N 192 on one CTA for a conv: a ragged last N tile (K = 320)"""
    _, plan = run_conv("c192s", 2, 64, 14, 14, 320, 3, 3, 1, 1, LY.nchwxc(64, 64), LY.kcrs_yk_xc(320, 64, 64, 64),
                       LY.nchwxc(320, 64), torch.bfloat16, epi=True, act=1,
                       cfg={"path": alt.PATH_TC, "block_n": 192, "cta_pair": 2}, expect_path=alt.PATH_TC)
    assert plan["block_n"] == 192 and plan["cta_pair"] == 2


@pytest.mark.parametrize("sk", [2, 3])
def test_tc_tail_split(sk):
    """tail split (split_cluster = 2): whole waves of tiles unsplit, the last
    partial wave's tiles split sk ways; GEMM with 2.3 waves of CTA pairs and a
    conv with residual, against the oracle"""
    M = 128 * 2 * 170   # 170 pair tiles x 1 N tile: 2 full waves of 74 pairs + a tail of 22
    _, plan = run_gemm("tail%d" % sk, M, 256, 512, [], LY.transpose2(), [], torch.bfloat16, epi=True,
                       cfg={"path": alt.PATH_TC, "block_n": 256, "split_k": sk, "split_cluster": 2},
                       expect_path=alt.PATH_TC)
    assert plan["split_k"] == sk and plan["split_cluster"] == 2
    xp, wp, yp = LY.nchwxc(256, 64), LY.kcrs_yk_xc(512, 256, 256, 64), LY.nchwxc(512, 64)
    run_conv("tailc%d" % sk, 8, 256, 14, 14, 512, 3, 3, 1, 1, xp, wp, yp, torch.bfloat16, epi=True,
             res_p=LY.nchwxc(512, 64), act=1, cfg={"path": alt.PATH_TC, "block_n": 256, "split_k": sk,
                                                   "split_cluster": 2}, expect_path=alt.PATH_TC)


# ------------------------------------------------------- dilation (DIL) --
DIL = [  # name, N, C, H, W, K, R, V, pad, dil, groups, x, w, y
    ("d2_nchw8c", 2, 16, 13, 11, 24, 3, 1, 2, 2, 1, LY.nchwxc(16, 8), LY.kcrs_yk_xc(24, 16, 8, 8), LY.nchwxc(24, 8)),
    ("d3_s2_plain", 1, 8, 17, 15, 8, 3, 2, 3, 3, 1, [], [], []),
    ("d2_grouped", 2, 16, 9, 9, 16, 3, 1, 2, 2, 4, LY.nhwc(), [], LY.nhwc()),
]


@pytest.mark.parametrize("case", DIL, ids=[c[0] for c in DIL])
@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
def test_dilated_conv(case, dtype):
    """dilated conv (the paper's DIL operator) through any layouts, on the SIMT
    path and (channel-tiled bf16 layouts) the tensor-core path"""
    name, N, C, H, W, K, R, V, pad, d, g, xp, wp, yp = case
    x = synth.activations(name + "x", (N, C, H, W))
    w = synth.weights(name + "w", (K, C // g, R, R))
    Ho = (H + 2 * pad - d * (R - 1) - 1) // V + 1
    Wo = (W + 2 * pad - d * (R - 1) - 1) // V + 1
    Ox, xph, xd = make_operand(name, xp, x, dtype)
    Ow, wph, wd = make_operand(name + "w", wp, w, dtype)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((N, K, Ho, Wo), yp)
    y = torch.full(Ly.phys_shape, 3.0, dtype=dtype, device="cuda")
    p = alt.conv_params(N, C, H, W, K, R, R, V, pad, g, dilation=d)
    pd = dict(N=N, C=C, H=H, W=W, K=K, R=R, S=R, stride_h=V, stride_w=V, pad_h=pad, pad_w=pad, groups=g,
              dil_h=d, dil_w=d)
    ref = oracle.conv2d(pd, Ox, xph, Ow, wph, act=1)
    paths = [alt.PATH_SIMT] + ([alt.PATH_TC] if g == 1 and dtype == torch.bfloat16 and C % 8 == 0 and xp else [])
    for path in paths:
        y.fill_(3.0)
        alt.conv2d(p, Lx, xd, Lw, wd, Ly, y, act=1, cfg={"path": path})
        torch.cuda.synchronize()
        assert alt.last_plan()["path"] == path
        assert_parity(read_output(oracle.Layout((N, K, Ho, Wo), yp), y, dtype), ref, dtype)
    with pytest.raises(alt.AltError) as e:   # forced depthwise path: no dilated kernel
        alt.conv2d(p, Lx, xd, Lw, wd, Ly, y, cfg={"path": alt.PATH_DW})
    assert e.value.code == alt._alt.ALT_E_UNSUPPORTED


# --------------------------------------------------- grouped conv (GRP) --
GRP = [  # name, N, C, H, W, K, R, V, pad, groups, x, w, y, residual
    ("g2_c64", 2, 64, 14, 14, 64, 3, 1, 1, 2, LY.nchwxc(64, 32), LY.kcrs_yk_xc(64, 32, 32, 32), LY.nchwxc(64, 32),
     None),
    ("g4_s2_res", 2, 128, 15, 13, 256, 3, 2, 1, 4, LY.nchwxc(128, 32), LY.kcrs_yk_xc(256, 32, 64, 32),
     LY.nchwxc(256, 64), LY.nchwxc(256, 64)),
    ("g8_1x1_ragged", 3, 64, 9, 7, 192, 1, 1, 0, 8, LY.nchwxc(64, 8), LY.kcrs_yk_xc(192, 8, 8, 8), LY.nchwxc(192, 8),
     LY.nchwxc(192, 8)),
]


@pytest.mark.parametrize("case", GRP, ids=[c[0] for c in GRP])
def test_grouped_conv_tensor_core(case):
    """grouped conv (the paper's GRP operator) on the tensor-core path: one
    launch per group reading its channel slabs, weight rows and writing its
    output channels through the declared layouts"""
    name, N, C, H, W, K, R, V, pad, g, xp, wp, yp, rp = case
    _, plan = run_conv(name, N, C, H, W, K, R, R, V, pad, xp, wp, yp, torch.bfloat16, groups=g, epi=True,
                       res_p=rp, act=1, cfg={"path": alt.PATH_AUTO}, expect_path=alt.PATH_TC)


@pytest.mark.parametrize("yp_name", ["padded NCHW8c", "tiled unfold template", "padded NCHW64c"])
@pytest.mark.parametrize("pads_zero", [False, True])
def test_epilogue_writes_consumer_templates(yp_name, pads_zero):
    """A tensor-core conv writing its consumer's padded / overlapped-tile input
    layout (the fused conversion of Fig. 5b): the vectorised writer stores
    every unfold copy; pad positions get 0 (pads_zero=False, buffer poisoned)
    or keep the zeros the caller guarantees (pads_zero=True, ALT_EPI_PADS_ZERO,
    zero buffer — padded layouts then go through the TMA-store epilogue)."""
    N, C, H, K = 2, 64, 14, 64
    yp = {"padded NCHW8c": LY.nchwxc(K, 8, pad_hw=1),
          "tiled unfold template": LY.conv_input_tiled(K, 16, H, H, 3, 3, 7, 7, 1, 1),
          "padded NCHW64c": LY.nchwxc(K, 64, pad_hw=1)}[yp_name]
    x = synth.activations("pzx", (N, C, H, H))
    w = synth.weights("pzw", (K, C, 3, 3))
    Xo, xph, xd = make_operand("pzx", LY.nchwxc(C, 64), x, torch.bfloat16)
    Wo_, wph, wd = make_operand("pzw", LY.kcrs_yk_xc(K, C, 64, 64), w, torch.bfloat16)
    Ly = alt.Layout((N, K, H, H), yp)
    fill = 0.0 if pads_zero else 3.0
    y = torch.full(Ly.phys_shape, fill, dtype=torch.bfloat16, device="cuda")
    p = alt.conv_params(N, C, H, H, K, 3, 3, 1, 1)
    alt.conv2d(p, alt.Layout(x.shape, LY.nchwxc(C, 64)), xd, alt.Layout(w.shape, LY.kcrs_yk_xc(K, C, 64, 64)), wd,
               Ly, y, act=1, cfg={"path": alt.PATH_TC}, pads_zero=pads_zero)
    torch.cuda.synchronize()
    assert alt.last_plan()["path"] == alt.PATH_TC
    ref = oracle.conv2d(dict(N=N, C=C, H=H, W=H, K=K, R=3, S=3, pad_h=1, pad_w=1), Xo, xph, Wo_, wph, act=1)
    got = read_output(oracle.Layout((N, K, H, H), yp), y, torch.bfloat16)
    assert_parity(got, ref, torch.bfloat16)


HALO_CASES = [
    # name, (N, C, H, W, K), cfg (tile with a W run of 16 / 32 / 64)
    ("14x14 tw16 bn64", (4, 64, 14, 14, 64), {"block_n": 64, "tile_n": 1, "tile_h": 8, "tile_w": 16}),
    ("28x28 tw32 bn128", (2, 128, 28, 28, 128), {"block_n": 128, "cta_pair": 2, "tile_n": 1, "tile_h": 4, "tile_w": 32}),
    ("56x56 tw64 pair", (2, 64, 56, 56, 128), {"block_n": 128, "tile_n": 1, "tile_h": 2, "tile_w": 64}),
    ("56x56 tw64 bn256 pair", (2, 64, 56, 56, 256), {"block_n": 256, "tile_n": 2, "tile_h": 1, "tile_w": 64}),
    ("ragged 13x13 tw16 residual", (3, 64, 13, 13, 64), {"block_n": 64, "tile_n": 2, "tile_h": 4, "tile_w": 16}),
]


@pytest.mark.parametrize("pad_x", [0, 1], ids=["oob-pad", "materialised-pad"])
@pytest.mark.parametrize("case", HALO_CASES, ids=[c[0] for c in HALO_CASES])
def test_tc_conv_halo(case, pad_x):
    """halo mode for stride-1 3x3 (block_k = 1 requests it): each input row
    segment is loaded once per filter row and the three taps along W read it
    at row offsets 0 / 1 / 2 (descriptor shift); vs the oracle"""
    name, (N, C, H, W, K), cfg = case
    res = LY.nchwxc(K, 64) if "residual" in name else None
    _, plan = run_conv("halo" + name, N, C, H, W, K, 3, 3, 1, 1, LY.nchwxc(C, 64, pad_hw=pad_x),
                       LY.kcrs_yk_xc(K, C, min(K, cfg["block_n"]), 64), LY.nchwxc(K, 64), torch.bfloat16, epi=True,
                       res_p=res, act=1, cfg={"path": alt.PATH_TC, "block_k": 1, **cfg}, expect_path=alt.PATH_TC)
    assert plan["block_k"] in (1, 3), plan   # a halo plan ran (3: the 2-D form, when eligible)


HALO2D_CASES = [
    # name, (N, C, H, W, K), cfg: one 64-channel slab, BLOCK_N 64, one image per tile
    ("56x56 tw64 th2", (2, 64, 56, 56, 64), {"block_n": 64, "tile_n": 1, "tile_h": 2, "tile_w": 64}),
    ("28x28 tw32 th4", (3, 64, 28, 28, 64), {"block_n": 64, "tile_n": 1, "tile_h": 4, "tile_w": 32}),
    ("ragged 13x13 tw16 th8", (2, 64, 13, 13, 64), {"block_n": 64, "tile_n": 1, "tile_h": 8, "tile_w": 16}),
    ("20x20 residual", (2, 64, 20, 20, 64), {"block_n": 64, "tile_n": 1, "tile_h": 4, "tile_w": 32}),
    ("C40 28x28", (2, 40, 28, 28, 64), {"block_n": 64, "tile_n": 1, "tile_h": 4, "tile_w": 32}),
]


@pytest.mark.parametrize("pad_x", [0, 1], ids=["oob-pad", "materialised-pad"])
@pytest.mark.parametrize("case", HALO2D_CASES, ids=[c[0] for c in HALO2D_CASES])
def test_tc_conv_halo2d(case, pad_x):
    """2-D halo (C <= 64, K <= 64, BLOCK_N 64): one box of (tile_h + 2) x
    tile_w input rows per tile, the nine taps read it at row offsets
    r tile_w + s, weights resident; vs the oracle"""
    name, (N, C, H, W, K), cfg = case
    res = LY.nchwxc(K, 8) if "residual" in name else None
    xp = LY.nchwxc(C, 64, pad_c=64 - C, pad_hw=pad_x) if C < 64 else LY.nchwxc(C, 64, pad_hw=pad_x)
    _, plan = run_conv("halo2d" + name, N, C, H, W, K, 3, 3, 1, 1, xp,
                       LY.kcrs_yk_xc(K, C, 64, 64, pad_c=64 - C) if C < 64 else LY.kcrs_yk_xc(K, C, 64, 64),
                       LY.nchwxc(K, 64), torch.bfloat16, epi=True,
                       res_p=res, act=1, cfg={"path": alt.PATH_TC, "block_k": 1, **cfg}, expect_path=alt.PATH_TC)
    assert plan["block_k"] == 3, plan   # the 2-D halo plan ran


@pytest.mark.parametrize("tile", [(4, 32), (2, 64), (8, 16)])
@pytest.mark.parametrize("W", [8, 26])
def test_tc_conv_single_output_row(tile, W):
    """Ho = 1 (stride 2, H = 4) with output tiles of several rows: y's size-1
    H dim drops out of the store view, so the warps whose 32-row sub-box lies
    past Ho must not store (they used to land on row 0; found by the
    randomized stress, seeds 842 / 844)"""
    th, tw = tile
    run_conv(f"ho1{th}{W}", 2, 32, 4, W, 64, 3, 3, 2, 0, LY.nchwxc(32, 32), LY.kcrs_yk_xc(64, 32, 64, 32),
             LY.nchwxc(64, 64), torch.bfloat16, epi=True, act=1,
             cfg={"path": alt.PATH_TC, "block_n": 64, "cta_pair": 2, "tile_n": 1, "tile_h": th, "tile_w": tw},
             expect_path=alt.PATH_TC)


def test_tc_conv_halo_request_with_paper_weight_order():
    """halo requested (block_k 1) with the paper's weight order i't o't (an
    MN-major B): the halo modes cannot issue MN-major B groups, so the plan
    falls back to the plain tap loop instead of writing past the B stage (an
    illegal address found by the randomized stress, seed 499)"""
    _, plan = run_conv("halopaperw", 3, 64, 28, 18, 280, 3, 3, 1, 1, LY.nhwc(), LY.kcrs_paper(280, 64, 8, 64),
                       LY.nchwxc(280, 8), torch.bfloat16, epi=True, act=1,
                       cfg={"path": alt.PATH_TC, "block_n": 64, "cta_pair": 2, "tile_n": 4, "tile_h": 1,
                            "tile_w": 32, "block_k": 1}, expect_path=alt.PATH_TC)
    assert plan["block_k"] == 64, plan


def test_tc_grouped_conv_misaligned_group_weight_offset():
    """grouped conv whose per-group weight offset (K / groups = 144) is not a
    multiple of the weight layout's k tile (32): the tensor-core plan is
    refused (its B box would start mid-tile and read the wrong rows — found by
    the randomized stress) and the automatic path stays exact"""
    args = ("grpmis", 2, 64, 12, 12, 288, 1, 1, 1, 0, LY.nchwxc(64, 8), LY.kcrs_yk_xc(288, 32, 32, 8),
            LY.nchwxc(288, 8), torch.bfloat16)
    with pytest.raises(alt.AltError) as e:
        run_conv(*args, groups=2, cfg={"path": alt.PATH_TC, "block_n": 64, "cta_pair": 2})
    assert e.value.code == alt._alt.ALT_E_UNSUPPORTED
    run_conv(*args, groups=2, cfg={"path": alt.PATH_AUTO})
    # aligned offsets (K / groups = 160 = 5 x 32) keep the tensor cores
    run_conv("grpal", 2, 64, 12, 12, 320, 1, 1, 1, 0, LY.nchwxc(64, 8), LY.kcrs_yk_xc(320, 32, 32, 8),
             LY.nchwxc(320, 8), torch.bfloat16, groups=2, cfg={"path": alt.PATH_TC, "block_n": 64, "cta_pair": 2},
             expect_path=alt.PATH_TC)


def _divs(n, cands):
    return [c for c in cands if n % c == 0]


@pytest.mark.parametrize("seed", range(300))
def test_tc_conv_random(seed):
    """random tensor-core convs: shape (ragged channels, small / odd images,
    stride 1 / 2, 1x1 / 3x3, padding), layouts (NCHW[x]c, padded, NHWC for x
    and y; KCRS[y]k[x]c / KRSC for w), kernel configuration (BLOCK_N, CTA
    pair, output-pixel tile, split-K, halo, residual, activation) drawn at
    random; vs the oracle (normwise + per-element bound).  Configurations the
    planner cannot serve on the tensor cores are skipped (ALT_E_UNSUPPORTED)."""
    import random
    rng = random.Random(7000 + seed)
    C = 8 * rng.randint(1, 12)
    K = 8 * rng.randint(1, 40)
    N = rng.randint(1, 4)
    H, W = rng.randint(4, 30), rng.randint(4, 30)
    R = rng.choice([1, 3])
    V = rng.choice([1, 1, 2])
    pad = rng.randint(0, R // 2)
    g = rng.choice([1, 1, 1, 2]) if C % 16 == 0 and K % 16 == 0 else 1     # grouped (GRP)
    dil = rng.choice([1, 1, 2]) if R == 3 and H >= 7 and W >= 7 else 1    # dilated (DIL)
    xc = rng.choice(_divs(C, (8, 16, 32, 64)))
    # plain NCHW (MN-major A: 1x1 unpadded convs with 8-multiple H W) and the
    # paper's weight order i't o't (MN-major B) join the K-major layouts
    xp = rng.choice([LY.nchwxc(C, xc), LY.nchwxc(C, xc, pad_hw=pad) if pad else LY.nchwxc(C, xc), LY.nhwc(), []])
    Cg = C // g
    wy, wx = rng.choice(_divs(K, (8, 16, 32, 64, 128, 256))), rng.choice(_divs(Cg, (8, 16, 32, 64)))
    wp = rng.choice([LY.kcrs_yk_xc(K, Cg, wy, wx), [("reorder", [0, 2, 3, 1])],
                     LY.kcrs_paper(K, Cg, rng.choice(_divs(K, (8, 16, 32, 64))), wx)])
    yc = rng.choice(_divs(K, (8, 16, 32, 64)))
    yp = rng.choice([LY.nchwxc(K, yc), LY.nhwc()])
    res = rng.choice([None, None, LY.nchwxc(K, yc)])
    cfg = {"path": alt.PATH_TC, "block_n": rng.choice([64, 128, 256]), "cta_pair": rng.choice([0, 2])}
    if rng.random() < 0.5:
        tw = rng.choice([4, 8, 16, 32, 64])
        th = rng.choice([t for t in (1, 2, 4, 8) if t * tw <= 128])
        cfg.update(tile_n=128 // (th * tw), tile_h=th, tile_w=tw)
    if rng.random() < 0.25:
        cfg["split_k"] = rng.choice([2, 3, 4])
        cfg["split_cluster"] = rng.choice([0, 1, 2])  # workspace / cluster DSMEM / tail split
    if R == 3 and V == 1 and rng.random() < 0.3:
        cfg["block_k"] = 1
    dtype = torch.float32 if rng.random() < 0.1 else torch.bfloat16  # fp32: three bf16 planes
    if dtype == torch.float32:
        cfg.pop("split_k", None)
        cfg.pop("split_cluster", None)
    if N == 1 and cfg.get("tile_n", 1) > 1:
        cfg.update(tile_n=1, tile_h=min(128 // cfg["tile_w"], 8), tile_w=128 // min(128 // cfg["tile_w"], 8))
    try:
        run_conv(f"rnd{seed}", N, C, H, W, K, R, R, V, pad, xp, wp, yp, dtype, epi=True, groups=g, dil=dil,
                 res_p=res, act=rng.choice([0, 1, 2]), cfg=cfg, expect_path=alt.PATH_TC)
    except alt.AltError as e:
        if e.code != alt._alt.ALT_E_UNSUPPORTED:
            raise
        # this configuration has no tensor-core plan (e.g. cluster split-K with
        # a residual): the automatic path must still be exact
        run_conv(f"rnd{seed}", N, C, H, W, K, R, R, V, pad, xp, wp, yp, dtype, epi=True, groups=g, dil=dil,
                 res_p=res, act=1, cfg={"path": alt.PATH_AUTO})


@pytest.mark.parametrize("seed", range(150))
def test_tc_gemm_random(seed):
    """random tensor-core GEMMs: ragged M / N / K, A in MK / KM / tiled
    M/mt K/kt mt kt, B in KN / NK / tiled N/nt K/kt nt kt / the paper's
    K/kt N/nt kt nt / NKn, C in MN / tiled, random BLOCK_N, CTA pair, split-K
    (bf16 and the fp32 three-plane path); vs the oracle"""
    import random
    rng = random.Random(9000 + seed)
    M = 8 * rng.randint(1, 80)
    N = 8 * rng.randint(1, 60)
    K = 8 * rng.randint(1, 60)
    ap = rng.choice([[], LY.transpose2()] + ([LY.gemm_a_tiled(M, K, mt, kt) for mt in _divs(M, (64, 128))
                                               for kt in _divs(K, (32, 64))][:1]))
    bps = [[], LY.transpose2()]
    bps += [LY.gemm_b_tiled_nk(K, N, nt, kt) for nt in _divs(N, (64, 128, 256)) for kt in _divs(K, (32, 64))][:1]
    bps += [LY.gemm_b_tiled_kn(K, N, kt, nt) for nt in _divs(N, (64, 128)) for kt in _divs(K, (32, 64))][:1]
    bps += [LY.gemm_nkn_b(K, N)] if N % 16 == 0 else []
    bp = rng.choice(bps)
    cp = rng.choice([[]] + [LY.gemm_c_tiled(M, N, mt, nt) for mt in _divs(M, (64, 128)) for nt in _divs(N, (64,))][:1])
    cfg = {"path": alt.PATH_TC, "block_n": rng.choice([64, 128, 192, 256]), "cta_pair": rng.choice([0, 2])}
    if cfg["block_n"] == 192 and N % 8:
        cfg["block_n"] = 128
    dtype = torch.float32 if rng.random() < 0.1 else torch.bfloat16
    if dtype == torch.bfloat16 and rng.random() < 0.2:
        cfg["split_k"] = rng.choice([2, 3])
    try:
        run_gemm(f"rg{seed}", M, N, K, ap, bp, cp, dtype, epi=True, cfg=cfg, expect_path=alt.PATH_TC)
    except alt.AltError as e:
        if e.code != alt._alt.ALT_E_UNSUPPORTED:
            raise
        # no tensor-core plan for these layouts: the automatic path (CUDA
        # cores) must still be exact
        run_gemm(f"rg{seed}", M, N, K, ap, bp, cp, dtype, epi=True, cfg={"path": alt.PATH_AUTO})


@pytest.mark.parametrize("seed", range(200))
def test_conv_random_any_path(seed):
    """random convs through the whole operator surface on the automatic path
    and, when it applies, each forced path (tensor cores, CUDA cores,
    depthwise): groups (1, 2, depthwise), dilation, stride, padding, the
    paper's tiled input / output templates and weight order, padded and
    plain layouts, fp32 / bf16; vs the oracle"""
    import random
    rng = random.Random(11000 + seed)
    dtype = torch.float32 if rng.random() < 0.3 else torch.bfloat16
    g = rng.choice([1, 1, 1, 2, "dw"])
    C = 8 * rng.randint(1, 8)
    K = C if g == "dw" else 8 * rng.randint(1, 8)
    groups = C if g == "dw" else g
    N, H, W = rng.randint(1, 3), rng.randint(5, 24), rng.randint(5, 24)
    R = rng.choice([1, 3]) if g != "dw" else 3
    V = rng.choice([1, 1, 2])
    d = rng.choice([1, 1, 2]) if g != "dw" else 1
    pad = rng.randint(0, d * (R // 2))
    Ho, Wo = (H + 2 * pad - d * (R - 1) - 1) // V + 1, (W + 2 * pad - d * (R - 1) - 1) // V + 1
    if Ho < 1 or Wo < 1:
        pytest.skip("empty output")
    it = rng.choice(_divs(C, (8, 16)))
    xps = [[], LY.nhwc(), LY.nchwxc(C, it)]
    if d == 1 and groups == 1:  # (R < V: a lossy template, reading A32)
        ht, wt = rng.choice([1, 2, 4]), rng.choice([1, 2, 4])
        if V * (ht - 1) + R <= H + 2 * pad and V * (wt - 1) + R <= W + 2 * pad:
            xps.append(LY.conv_input_tiled(C, it, H, W, R, R, ht, wt, V, pad))
    xp = rng.choice(xps)
    wps = [[], [("reorder", [0, 2, 3, 1])]]
    if groups == 1:
        wps += [LY.kcrs_yk_xc(K, C, rng.choice(_divs(K, (8, 16))), it), LY.kcrs_paper(K, C, rng.choice(_divs(K, (8, 16))), it)]
    if g == "dw":
        wps = [[("reorder", [1, 2, 3, 0])], []]
    wp = rng.choice(wps)
    ot = rng.choice(_divs(K, (8, 16)))
    yps = [[], LY.nhwc(), LY.nchwxc(K, ot), LY.nchwxc(K, ot, pad_hw=rng.randint(1, 2))]
    for ht2 in (2, 4):
        if Ho % ht2 == 0 and Wo % ht2 == 0:
            yps.append(LY.conv_output_tiled(K, ot, Ho, Wo, ht2, ht2))
    # the next 3x3 layer's input template (pad + unfold: the epilogue writes
    # every overlapped copy and the pad zeros; checked by read_output)
    ht3 = rng.choice([t for t in (1, 2, 4) if t <= Ho])
    wt3 = rng.choice([t for t in (1, 2, 4) if t <= Wo])
    yps.append(LY.conv_input_tiled(K, ot, Ho, Wo, 3, 3, ht3, wt3, 1, 1))
    yp = rng.choice(yps)
    x = synth.activations(f"ra{seed}x", (N, C, H, W))
    w = synth.weights(f"ra{seed}w", (K, C // groups, R, R))
    Ox, xph, xd = make_operand(f"ra{seed}", xp, x, dtype)
    Ow, wph, wd = make_operand(f"ra{seed}w", wp, w, dtype)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((N, K, Ho, Wo), yp)
    p = alt.conv_params(N, C, H, W, K, R, R, V, pad, groups, dilation=d)
    act = rng.choice([0, 1, 2])
    sc, bi = synth.bn_scale(f"ra{seed}s", K), synth.bn_bias(f"ra{seed}b", K)
    pd = dict(N=N, C=C, H=H, W=W, K=K, R=R, S=R, stride_h=V, stride_w=V, pad_h=pad, pad_w=pad, groups=groups,
              dil_h=d, dil_w=d)
    rp = rng.choice([None, None, [], LY.nchwxc(K, ot), LY.nhwc()])
    kw, ref_kw = {}, {}
    if rp is not None:  # residual add in the epilogue, read through its own layout
        r = synth.activations(f"ra{seed}r", (N, K, Ho, Wo))
        Ro, rph, rd = make_operand(f"ra{seed}r", rp, r, dtype)
        kw.update(residual=rd, residual_l=alt.Layout((N, K, Ho, Wo), rp))
        ref_kw.update(res_l=Ro, residual=rph)
    ref = oracle.conv2d(pd, Ox, xph, Ow, wph, act=act, scale=sc.double().numpy(), bias=bi.double().numpy(),
                        **ref_kw)
    ran = 0
    for path in (alt.PATH_AUTO, alt.PATH_TC, alt.PATH_SIMT, alt.PATH_DW):
        y = torch.full(Ly.phys_shape, 3.0, dtype=dtype, device="cuda")
        try:
            alt.conv2d(p, Lx, xd, Lw, wd, Ly, y, scale=sc.cuda(), bias=bi.cuda(), act=act, cfg={"path": path},
                       **kw)
        except alt.AltError as e:
            assert path != alt.PATH_AUTO and e.code == alt._alt.ALT_E_UNSUPPORTED, e
            continue
        torch.cuda.synchronize()
        assert_parity(read_output(oracle.Layout((N, K, Ho, Wo), yp), y, dtype), ref, dtype)
        ran += 1
    assert ran >= 2   # the automatic path plus at least the path it picked
