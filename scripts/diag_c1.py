"""R18 conv1 (b256, window-folded input) parity per tile config, with the error pattern."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from tests.helpers import norm_rel, words
ch = (CH.mobilenet_v2 if sys.argv[2] == "mv2" else CH.resnet18)(int(sys.argv[1]), torch.device("cuda", 0))
N = ch.N
op = ch.ops[0]
L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
wl, w, sc, bi = ch.weights[0]
alt.relayout(ch.img_plain, ch.img, ch.layouts["img"], ch.buf["img"])
torch.cuda.synchronize()
p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
shp = lambda t: (1,) + tuple(ch.shapes[t][1:])
Ox = oracle.Layout(shp(src), ch.layouts[src].prims); Ow = oracle.Layout(wl.logical_shape, wl.prims)
pd = dict(N=1, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride, stride_w=L.stride, pad_h=L.pad, pad_w=L.pad)
refs = {n: oracle.conv2d(pd, Ox, words(ch.buf[src][n:n+1]), Ow, words(w), scale=sc.double().cpu().numpy(),
                         bias=bi.double().cpu().numpy(), act=2 if sys.argv[2] == "mv2" else 1) for n in (0, 1, N - 1)}
Oy = oracle.Layout(shp(dst), ch.layouts[dst].prims)
tl = [(16, 2, 4), (8, 4, 4), (8, 1, 16), (2, 8, 8), (32, 1, 4), (4, 4, 8), (16, 1, 8), (1, 4, 32)]
for cfg in [None] + [{"path": 1, "block_n": 64, "cta_pair": 2, "tile_n": a, "tile_h": b, "tile_w": c} for (a, b, c) in tl for _ in range(2)]:
    ch.buf[dst].fill_(7.0)
    alt.conv2d(p, ch.layouts[src], ch.buf[src], wl, w, ch.layouts[dst], ch.buf[dst], scale=sc, bias=bi, act="relu6" if sys.argv[2] == "mv2" else "relu", cfg=cfg)
    torch.cuda.synchronize()
    out = []
    for n, ref in refs.items():
        got = Oy.read_f64(words(ch.buf[dst][n:n+1]))
        e = np.abs(got - ref)
        bad = np.argwhere(e > 0.05 * (np.abs(ref).max()))
        out.append((n, round(norm_rel(got, ref), 4), len(bad), bad[:3].tolist()))
    pl = alt.last_plan()
    print((pl["tile_n"], pl["tile_h"], pl["tile_w"]), out, flush=True)
