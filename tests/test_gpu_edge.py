"""Edge cases on the GPU: empty batches are no-ops, ragged shapes (odd spatial
extents, output channels that are not a multiple of BLOCK_N, batch 1) match
the oracle on every path."""
import numpy as np
import pytest
import torch

import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from tests.test_gpu_conv import run_conv, run_gemm

pytestmark = pytest.mark.gpu


def test_empty_batch_conv_and_gemm_are_noops():
    Lx, Lw, Ly = alt.Layout((1, 16, 8, 8), []), alt.Layout((32, 16, 3, 3), []), alt.Layout((1, 32, 8, 8), [])
    x = torch.zeros(1, 16, 8, 8, dtype=torch.bfloat16, device="cuda")
    w = torch.zeros(32, 16, 3, 3, dtype=torch.bfloat16, device="cuda")
    y = torch.full((1, 32, 8, 8), 5.0, dtype=torch.bfloat16, device="cuda")
    n0 = alt.launch_count()
    alt.conv2d(alt.conv_params(0, 16, 8, 8, 32, 3, 3, 1, 1), Lx, x, Lw, w, Ly, y)
    La, Lb, Lc = alt.Layout((4, 16), []), alt.Layout((16, 8), []), alt.Layout((4, 8), [])
    c = torch.full((4, 8), 5.0, dtype=torch.bfloat16, device="cuda")
    alt.matmul(0, 8, 16, La, torch.zeros(4, 16, dtype=torch.bfloat16, device="cuda"), Lb,
               torch.zeros(16, 8, dtype=torch.bfloat16, device="cuda"), Lc, c)
    torch.cuda.synchronize()
    assert alt.launch_count() == n0              # nothing launched
    assert bool((y == 5.0).all()) and bool((c == 5.0).all())   # nothing written


RAGGED = [  # name, N, C, H, W, K, R, V, pad, x, w, y
    ("odd_hw_k40", 3, 24, 13, 11, 40, 3, 1, 1, LY.nchwxc(24, 8), LY.kcrs_yk_xc(40, 24, 8, 8), LY.nchwxc(40, 8)),
    ("b1_s2_k72", 1, 64, 15, 9, 72, 3, 2, 1, LY.nchwxc(64, 64), LY.kcrs_yk_xc(72, 64, 8, 64), LY.nchwxc(72, 8)),
    ("k200_bn256", 2, 32, 7, 7, 200, 1, 1, 0, LY.nchwxc(32, 32), LY.kcrs_yk_xc(200, 32, 8, 32), LY.nchwxc(200, 8)),
]


@pytest.mark.parametrize("case", RAGGED, ids=[c[0] for c in RAGGED])
@pytest.mark.parametrize("path", [alt.PATH_AUTO, alt.PATH_SIMT])
def test_ragged_shapes(case, path):
    name, N, C, H, W, K, R, V, pad, xp, wp, yp = case
    run_conv("rg" + name, N, C, H, W, K, R, R, V, pad, xp, wp, yp, torch.bfloat16, epi=True, act=1,
             cfg={"path": path})


def test_ragged_gemm_rows_and_cols():
    """M not a multiple of 128, N not a multiple of BLOCK_N, K not a multiple of 64"""
    run_gemm("rgg", 300, 200, 136, [], LY.transpose2(), [], torch.bfloat16, epi=True, cfg={"path": alt.PATH_AUTO})
