"""fp32 conv / GEMM on the tensor cores (reading A27, csrc/split3.cu): each
fp32 operand is split into three bf16 planes and the six plane products of
weight > 2^-24 run as tcgen05 MMAs with fp32 accumulation.  BASELINE's fp32
bar: max |y - ref| / max |ref| <= 1e-5 against the fp64 oracle, on every
layout family the bf16 path takes (the split reads any layout), with the
fused epilogue and an fp32 residual, at sizes with several tiles and ragged
tails, and at a full ResNet-50 layer."""
import numpy as np
import pytest
import torch

import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from tests.helpers import FP32_TOL
from tests.test_gpu_conv import run_conv, run_gemm

pytestmark = pytest.mark.gpu
TC = {"path": alt.PATH_TC}
F32 = torch.float32

CONV = [
    # name, (N, C, H, W, K, R, S, V, pad), x, w, y
    ("NCHW8c 3x3", (2, 64, 14, 14, 128, 3, 3, 1, 1), LY.nchwxc(64, 8), LY.kcrs_yk_xc(128, 64, 16, 8), LY.nchwxc(128, 16)),
    ("NCHW 1x1 (plain)", (3, 64, 13, 13, 96, 1, 1, 1, 0), [], [], []),
    ("NHWC 3x3 s2", (2, 32, 17, 15, 64, 3, 3, 2, 1), LY.nhwc(), [("reorder", [0, 2, 3, 1])], LY.nhwc()),
    ("C=3 7x7 s2 (conv1-like)", (2, 3, 32, 32, 64, 7, 7, 2, 3), [], [], LY.nchwxc(64, 64)),
    ("tiled unfold in / paper weights / tiled out", (2, 16, 14, 14, 32, 3, 3, 1, 1),
     LY.conv_input_tiled(16, 8, 14, 14, 3, 3, 7, 7, 1, 1), LY.kcrs_paper(32, 16, 16, 8),
     LY.conv_output_tiled(32, 16, 14, 14, 7, 7)),
    ("ragged K 40", (2, 24, 9, 11, 40, 3, 3, 1, 1), LY.nchwxc(24, 8), [], LY.nhwc()),
]


@pytest.mark.parametrize("case", CONV, ids=[c[0] for c in CONV])
def test_fp32_tc_conv(case):
    name, (N, C, H, W, K, R, S, V, pad), xp, wp, yp = case
    err, plan = run_conv("f32" + name, N, C, H, W, K, R, S, V, pad, xp, wp, yp, F32, epi=True, act=1, cfg=TC,
                         expect_path=alt.PATH_TC)
    assert err <= FP32_TOL


def test_fp32_tc_conv_residual_relu6():
    err, _ = run_conv("f32res", 2, 64, 12, 12, 64, 3, 3, 1, 1, LY.nchwxc(64, 16), LY.kcrs_yk_xc(64, 64, 64, 16),
                      LY.nchwxc(64, 32), F32, epi=True, res_p=LY.nhwc(), act=2, cfg=TC, expect_path=alt.PATH_TC)
    assert err <= FP32_TOL


def test_fp32_auto_takes_tensor_cores():
    _, plan = run_conv("f32auto", 1, 16, 14, 14, 32, 3, 3, 1, 1, LY.nchwxc(16, 8), LY.kcrs_yk_xc(32, 16, 16, 8),
                       LY.nchwxc(32, 16), F32)
    assert plan["path"] == alt.PATH_TC


GEMM = [
    ("MK/KN/MN", 300, 192, 160, [], [], []),
    ("tiled template", 256, 128, 192, LY.gemm_a_tiled(256, 192, 64, 64), LY.gemm_b_tiled_kn(192, 128, 64, 64),
     LY.gemm_c_tiled(256, 128, 64, 64)),
    ("NKn", 256, 128, 192, [("split", 0, [16, 16]), ("reorder", [0, 2, 1])], LY.gemm_nkn_b(192, 128), []),
    ("ragged K 100", 130, 72, 100, [], LY.transpose2(), []),
]


@pytest.mark.parametrize("case", GEMM, ids=[c[0] for c in GEMM])
def test_fp32_tc_gemm(case):
    name, M, N, K, ap, bp, cp = case
    err, _ = run_gemm("f32g" + name, M, N, K, ap, bp, cp, F32, epi=True, cfg=TC, expect_path=alt.PATH_TC)
    assert err <= FP32_TOL


@pytest.mark.parametrize("cfg", [{"block_n": 256}, {"block_n": 128, "cta_pair": 2}, {"block_n": 64, "split_k": 2}])
def test_fp32_tc_kernel_configs(cfg):
    err, _ = run_conv("f32cfg", 2, 128, 14, 14, 256, 3, 3, 1, 1, LY.nchwxc(128, 64), LY.kcrs_yk_xc(256, 128, 256, 64),
                      LY.nchwxc(256, 64), F32, epi=True, act=1, cfg={**TC, **cfg}, expect_path=alt.PATH_TC)
    assert err <= FP32_TOL


def test_fp32_tc_r50_layer_full_size():
    """ResNet-50 l3.3x3 (256 -> 256, 14x14) at batch 32 in fp32: the whole
    output against the oracle"""
    err, _ = run_conv("f32l3", 32, 256, 14, 14, 256, 3, 3, 1, 1, LY.nchwxc(256, 64), LY.kcrs_yk_xc(256, 256, 256, 64),
                      LY.nchwxc(256, 64), F32, epi=True, act=1, cfg=TC, expect_path=alt.PATH_TC)
    assert err <= FP32_TOL


def test_fp32_r50_layer_set_b32_bench_config():
    """the R50 set at batch 32 in fp32 exactly as bench.py's aux.r50_fp32 runs
    it (layouts and kernel configurations from the tune cache, split-K forms
    dropped): every image of every layer against the oracle at the fp32 bar"""
    import oracle
    import bench
    from tests.helpers import norm_rel, words
    S = bench.LayerSet(32, torch.device("cuda", 0), F32)
    S.step()
    torch.cuda.synchronize()
    for l in S.layers:
        L = l["L"]
        Ho, Wo = L.out_hw()
        Ox = oracle.Layout((32, L.C, L.H, L.W), l["lx"].prims)
        Ow = oracle.Layout((L.K, L.C, L.R, L.S), l["lw"].prims)
        Oy = oracle.Layout((32, L.K, Ho, Wo), l["ly"].prims)
        pd = dict(N=32, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride, stride_w=L.stride,
                  pad_h=L.pad, pad_w=L.pad)
        ref = oracle.conv2d_f64(pd, Ox.read_f64(words(l["x"])), Ow.read_f64(words(l["w"])),
                                l["sc"].double().cpu().numpy(), l["bi"].double().cpu().numpy(), None, 1)
        yw = words(l["y"])
        assert Oy.check_consistent(yw) == 0, L.name
        got = Oy.read_f64(yw)
        for n in range(32):
            assert norm_rel(got[n], ref[n]) <= FP32_TOL, (L.name, n, l["cfg"])
