"""Tensor-core parity for MN-major operands: layouts
whose stride-1 dim is the M (pixel / row) or N (output-channel / column) run
instead of the reduction run — the GEMM default KN B and the NKn layouts of
§2 (reading A12), the paper's GEMM template B K/kt N/nt kt nt
(P:1152-1179), the paper's weight order i't o't and the plain
NCHW activation — read by tcgen05 MMA with the MN-major smem descriptor
(no conversion).  Every case must run on the tensor-core path (path 1) and
meet the bf16 normwise bar against the fp64 oracle."""
import pytest
import torch

import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from tests.test_gpu_conv import run_conv, run_gemm

pytestmark = pytest.mark.gpu

TC = {"path": alt.PATH_TC}


def _nkn_a(M):
    return [("split", 0, [M // 16, 16]), ("reorder", [0, 2, 1])]


GEMM_MN = [
    # name, M, N, K, A, B, C, cfg
    ("MK/KN(row B)/MN", 300, 192, 160, [], [], [], {}),
    ("MK/KN/MN bn128 single", 256, 128, 192, [], [], [], {"block_n": 128, "cta_pair": 2}),
    ("KM(col A)/NK/MN", 256, 128, 192, LY.transpose2(), LY.transpose2(), [], {}),
    ("KM/KN both MN-major", 384, 256, 128, LY.transpose2(), [], [], {}),
    ("NKn (A12)", 256, 128, 192, _nkn_a(256), LY.gemm_nkn_b(192, 128), LY.gemm_c_tiled(256, 128, 16, 16), {}),
    ("template B K/kt N/nt kt nt", 256, 256, 192, LY.gemm_a_tiled(256, 192, 64, 64),
     LY.gemm_b_tiled_kn(192, 256, 64, 128), LY.gemm_c_tiled(256, 256, 64, 64), {}),
    ("template B nt 32", 256, 128, 128, [], LY.gemm_b_tiled_kn(128, 128, 64, 32), [], {"block_n": 64}),
    ("KN bn64 split-K 2", 256, 64, 512, [], [], [], {"block_n": 64, "split_k": 2}),
]


@pytest.mark.parametrize("case", GEMM_MN, ids=[c[0] for c in GEMM_MN])
def test_tc_gemm_mn_major(case):
    name, M, N, K, ap, bp, cp, cfg = case
    run_gemm("mn" + name, M, N, K, ap, bp, cp, torch.bfloat16, epi=True, cfg={**TC, **cfg},
             expect_path=alt.PATH_TC)


# TMA needs every global stride to be a multiple of 16 bytes, so plain NCHW
# reaches the tensor cores when W and H*W are multiples of 8 (bf16): W = 16,
# 24, 32, 56, 112 ... (R50 stage 1: 56x56), and a box must start 16-byte
# aligned along the stride-1 dim, so an MN-major activation serves 1x1
# unpadded convs; NCHW 3x3 and W = 28 / 14 / 7 run on the CUDA-core path
# (test_nchw_falls_back).  MN-major weights (the paper's i't o't) take any
# filter size.
CONV_MN = [
    # name, (N, C, H, W, K, R, S, V, pad), x, w, y, cfg
    ("NCHW 1x1", (3, 64, 16, 16, 64, 1, 1, 1, 0), [], LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64), {}),
    ("NCHW 1x1 W=24 ragged", (2, 32, 12, 24, 64, 1, 1, 1, 0), [], LY.kcrs_yk_xc(64, 32, 64, 32), LY.nhwc(), {}),
    ("NCHW 56x56 1x1 (R50 l1)", (2, 64, 56, 56, 256, 1, 1, 1, 0), [], LY.kcrs_yk_xc(256, 64, 256, 64),
     LY.nchwxc(256, 64), {}),
    ("NCHW in/out 1x1", (2, 64, 16, 16, 64, 1, 1, 1, 0), [], LY.kcrs_yk_xc(64, 64, 64, 64), [], {}),
    ("NCHW 1x1 W=8", (4, 64, 8, 8, 128, 1, 1, 1, 0), [], LY.kcrs_yk_xc(128, 64, 128, 64), LY.nchwxc(128, 64), {}),
    ("NCHW 1x1 single CTA bn64", (2, 128, 16, 32, 64, 1, 1, 1, 0), [], LY.kcrs_yk_xc(64, 128, 64, 64),
     LY.nchwxc(64, 64), {"block_n": 64}),
    ("paper weights i't o't 64", (2, 64, 14, 14, 128, 3, 3, 1, 1), LY.nchwxc(64, 64), LY.kcrs_paper(128, 64, 64, 64),
     LY.nchwxc(128, 64), {}),
    ("paper weights i't o't 32 bn64", (2, 64, 14, 14, 64, 3, 3, 1, 1), LY.nchwxc(64, 32),
     LY.kcrs_paper(64, 64, 32, 32), LY.nchwxc(64, 32), {"block_n": 64}),
    ("paper weights stride 2", (2, 64, 16, 16, 128, 3, 3, 2, 1), LY.nchwxc(64, 64), LY.kcrs_paper(128, 64, 64, 64),
     LY.nchwxc(128, 64), {}),
    ("NCHW + paper weights (both MN)", (2, 64, 16, 16, 128, 1, 1, 1, 0), [], LY.kcrs_paper(128, 64, 64, 64),
     LY.nchwxc(128, 64), {}),
]


@pytest.mark.parametrize("case", CONV_MN, ids=[c[0] for c in CONV_MN])
def test_tc_conv_mn_major(case):
    name, (N, C, H, W, K, R, S, V, pad), xp, wp, yp, cfg = case
    run_conv("mn" + name, N, C, H, W, K, R, S, V, pad, xp, wp, yp, torch.bfloat16, epi=True, act=1,
             cfg={**TC, **cfg}, expect_path=alt.PATH_TC)


@pytest.mark.parametrize("shape", [(14, 1, 0), (16, 3, 1)], ids=["14x14 1x1 unaligned stride", "16x16 3x3 taps"])
def test_nchw_falls_back(shape):
    """NCHW at 14x14 (row stride 28 B is not a TMA stride) or with 3x3 taps
    along the stride-1 W dim: AUTO runs the CUDA-core path (exact), TC
    reports ALT_E_UNSUPPORTED"""
    H, R, pad = shape
    args = ("mnfb", 2, 64, H, H, 64, R, R, 1, pad, [], LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64),
            torch.bfloat16)
    _, plan = run_conv(*args)
    assert plan["path"] == alt.PATH_SIMT
    with pytest.raises(alt.AltError) as e:
        run_conv(*args, cfg=TC)
    assert e.value.code == alt._alt.ALT_E_UNSUPPORTED


def test_tc_conv_mn_major_residual():
    run_conv("mnres", 2, 64, 16, 16, 64, 1, 1, 1, 0, [], LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64),
             torch.bfloat16, epi=True, res_p=[], act=1, cfg=TC, expect_path=alt.PATH_TC)
