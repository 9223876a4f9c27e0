"""conv1 (7x7 s2, C=3, window-folded input) output-tile sweep at a batch."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, nets
from scripts.exptime import timeit
N = int(sys.argv[1]) if len(sys.argv) > 1 else 32
L = nets.RESNET50[0]
Ho, Wo = L.out_hw()
lx = alt.Layout((N, L.C, L.H, L.W), LY.conv_input_wfold(L.C, L.S, L.stride, L.pad))
lw = alt.Layout((L.K, L.C, L.R, L.S), LY.kcrs_wfold(L.K, L.C, L.S))
ly = alt.Layout((N, L.K, Ho, Wo), LY.nchwxc(L.K, 64))
xt = lx.empty(torch.bfloat16, "cuda").normal_(); wt = lw.empty(torch.bfloat16, "cuda").normal_()
yt = ly.empty(torch.bfloat16, "cuda")
sc = torch.ones(L.K, device="cuda"); bi = torch.zeros(L.K, device="cuda")
p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
res = []
for th in (1, 2, 4, 8, 16):
    for tw in (8, 16, 32, 64, 128):
        tn = 128 // (th * tw)
        if tn < 1 or tn > N: continue
        cfg = {"path": 1, "block_n": 64, "cta_pair": 2, "tile_n": tn, "tile_h": th, "tile_w": tw}
        try:
            us = timeit(lambda: alt.conv2d(p, lx, xt, lw, wt, ly, yt, scale=sc, bias=bi, act="relu", cfg=cfg))
            res.append((round(us, 1), tn, th, tw))
        except Exception as e:
            res.append((1e9, tn, th, tw, str(e)[:60]))
res.sort(key=lambda r: r[0])
print("conv1 N=%d" % N, res[:8])
