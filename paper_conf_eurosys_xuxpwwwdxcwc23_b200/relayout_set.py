"""The relayout bandwidth set (BASELINE config family D6): layout
conversions between the tensors of the paper's workloads at full size.
Algorithmic bytes = elem * (logical elements read + dst physical elements
written): pad zeros are written not read, unfold duplicates are written."""
from __future__ import annotations

from . import layouts as LY


def cases():
    N = 256
    return [
        ("R1 NCHW->NCHW8c", (N, 64, 56, 56), [], LY.nchwxc(64, 8)),
        ("R1 NCHW->NCHW16c", (N, 64, 56, 56), [], LY.nchwxc(64, 16)),
        ("R1 NCHW->NCHW32c", (N, 64, 56, 56), [], LY.nchwxc(64, 32)),
        ("R1 NCHW->NCHW64c", (N, 64, 56, 56), [], LY.nchwxc(64, 64)),
        ("R2 NCHW->NHWC", (N, 64, 56, 56), [], LY.nhwc()),
        ("R3 NCHW->pad+unfold(8x8)+NCHW8c", (N, 64, 56, 56), [],
         LY.conv_input_tiled(64, 8, 56, 56, 3, 3, 8, 8, 1, 1)),
        ("R4 NCHW8c->NCHW", (N, 64, 56, 56), LY.nchwxc(64, 8), []),
        ("R4 NHWC->NCHW", (N, 64, 56, 56), LY.nhwc(), []),
        ("R5 images NCHW->pad(C)+NCHW8c", (N, 3, 224, 224), [], LY.nchwxc(3, 8, pad_c=5)),
        ("R6 row-major->[M/128][K/64][128][64]", (8192, 3072), [], LY.gemm_a_tiled(8192, 3072, 128, 64)),
        ("R7 KCRS->KCRS16k16c", (512, 512, 3, 3), [], LY.kcrs_yk_xc(512, 512, 16, 16)),
        ("R8 images NCHW->window-folded conv1 input", (N, 3, 224, 224), [], LY.conv_input_wfold(3, 7, 2, 3)),
    ]


def alg_bytes(src_l, dst_l, esize):
    logical = 1
    for s in src_l.logical_shape:
        logical *= s
    return esize * (logical + dst_l.phys_numel)
