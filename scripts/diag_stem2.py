"""Isolate the MV2-stem failure: window-folded 3x3 s2 C=3 conv at several sizes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, synth
from tests.helpers import norm_rel, words, make_operand
CASES = [(16, 224, 32, 3, 2, 1, 3), (16, 112, 32, 3, 1, 1, 16), (16, 112, 64, 3, 1, 1, 16), (16, 112, 64, 1, 1, 0, 16),
         (16, 112, 64, 3, 1, 1, 32), (16, 112, 64, 3, 1, 1, 64)]
for (N, H, K, S, stride, pad, C) in CASES:
    x = synth.activations("st%d%d" % (N, H), (N, C, H, H)); w = synth.weights("stw%d" % S, (K, C, S, S))
    if C % 8:
        xp, wp = LY.conv_input_wfold(C, S, stride, pad), LY.kcrs_wfold(K, C, S)
    else:
        xp, wp = LY.nchwxc(C, C), LY.kcrs_yk_xc(K, C, K, C)
    yp = LY.nchwxc(K, 32 if K % 64 else 64)
    Ox, xph, xd = make_operand("x", xp, x, torch.bfloat16); Ow, wph, wd = make_operand("w", wp, w, torch.bfloat16)
    Ho = (H + 2 * pad - S) // stride + 1
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout((N, K, Ho, Ho), yp)
    p = alt.conv_params(N, C, H, H, K, S, S, stride, pad)
    pd = dict(N=1, C=C, H=H, W=H, K=K, R=S, S=S, stride_h=stride, stride_w=stride, pad_h=pad, pad_w=pad)
    Ox1, Oy1 = oracle.Layout((1, C, H, H), xp), oracle.Layout((1, K, Ho, Ho), yp)
    res = []
    for rep in range(2):
        y = torch.full(Ly.phys_shape, 3.0, dtype=torch.bfloat16, device="cuda")
        alt.conv2d(p, Lx, xd, Lw, wd, Ly, y)
        torch.cuda.synchronize()
        errs = []
        for n in sorted({0, N - 1}):
            ref = oracle.conv2d(pd, Ox1, words(xd[n:n+1]), Ow, wph)
            errs.append(round(norm_rel(Oy1.read_f64(words(y[n:n+1])), ref), 4))
        res.append(errs)
    pl = alt.last_plan()
    print((N, H, K, S, stride, pad), "E/Cp", Lx.phys_shape[-2:], "tile", (pl["tile_n"], pl["tile_h"], pl["tile_w"]), "bn", pl["block_n"], res, flush=True)
