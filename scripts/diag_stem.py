"""MV2 stem: image relayout (window-folded, K_ROW) bit-exactness vs the oracle, then the stem conv, repeated."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from tests.helpers import norm_rel, words
which = sys.argv[1]
ch = CH.mobilenet_v2(16, torch.device("cuda", 0)) if which == "mv2" else CH.resnet18(256, torch.device("cuda", 0))
N = ch.N
Si = oracle.Layout(ch.shapes["img"], [])
Di = oracle.Layout((1,) + tuple(ch.shapes["img"][1:]), ch.layouts["img"].prims)
imgw = words(ch.img)
for rep in range(3):
    ch.buf["img"].fill_(0)
    alt.relayout(ch.img_plain, ch.img, ch.layouts["img"], ch.buf["img"])
    torch.cuda.synchronize()
    bad = []
    for n in (0, 1, N // 2, N - 1):
        want = Di.materialize(imgw[n:n + 1])
        got = words(ch.buf["img"][n:n + 1]).reshape(want.shape)
        nd = int((got != want).sum())
        if nd: bad.append((n, nd, np.argwhere(got != want)[:3].tolist()))
    print("relayout rep", rep, "plan", ch.layouts["img"].phys_shape, "mismatching images:", bad, flush=True)
