"""One launch each of the HBM-bound kernels at benchmark sizes (for ncu):
K_ROW relayout (R8 window-folded images b256, R5, R3), MV2 depthwise, R18 pool."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, relayout_set
dev = torch.device("cuda", 0)
cases = {c[0][:2]: c for c in relayout_set.cases()}
for key in ("R8", "R5", "R3"):
    name, shape, sp, dp = cases[key]
    S, D = alt.Layout(shape, sp), alt.Layout(shape, dp)
    src = S.empty(torch.bfloat16, dev).normal_()
    dst = D.empty(torch.bfloat16, dev)
    alt.relayout(S, src, D, dst)
torch.cuda.synchronize()
# depthwise C144 56x56 b16 (MV2), vector weights
N, C, H = 16, 144, 56
lx = alt.Layout((N, C, H, H), LY.nchwxc(C, 16))
lw = alt.Layout((C, 1, 3, 3), [("reorder", [1, 2, 3, 0])])
x = lx.empty(torch.bfloat16, dev).normal_(); w = lw.empty(torch.bfloat16, dev).normal_(); y = lx.empty(torch.bfloat16, dev)
sc = torch.ones(C, device=dev); bi = torch.zeros(C, device=dev)
alt.conv2d(alt.conv_params(N, C, H, H, C, 3, 3, 1, 1, C), lx, x, lw, w, lx, y, scale=sc, bias=bi, act="relu6")
# R18 maxpool b256 64x112x112 -> 56x56
N, C, H = 256, 64, 112
lx = alt.Layout((N, C, H, H), LY.nchwxc(C, 64)); ly = alt.Layout((N, C, 56, 56), LY.nchwxc(C, 64))
x = lx.empty(torch.bfloat16, dev).normal_(); y = ly.empty(torch.bfloat16, dev)
alt.pool2d(alt.conv_params(N, C, H, H, C, 3, 3, 2, 1), lx, x, ly, y, "max")
torch.cuda.synchronize()
