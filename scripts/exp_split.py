"""Time R50 layers under kernel configs (bn, cta_pair, split_k) at batch 32."""
import sys
import torch
sys.path.insert(0, ".")
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, nets, synth
from scripts.exptime import timeit

N = 32
names = sys.argv[1].split(",")
cfgs = [(256, 0, 1), (256, 0, 2), (256, 0, 3), (256, 2, 1), (256, 2, 2), (256, 2, 4), (256, 2, 5), (256, 2, 6),
        (128, 1, 1), (128, 1, 2), (128, 2, 1), (128, 2, 2), (128, 2, 3), (128, 2, 4), (64, 2, 1), (64, 2, 2), (64, 2, 4)]
for L in nets.RESNET50:
    if L.name not in names:
        continue
    Ho, Wo = L.out_hw()
    x = min(L.C, 64)
    xp, yp = LY.nchwxc(L.C, x), LY.nchwxc(L.K, 64)
    lx, ly = alt.Layout((N, L.C, L.H, L.W), xp), alt.Layout((N, L.K, Ho, Wo), yp)
    xt = lx.empty(torch.bfloat16, "cuda").normal_()
    yt = ly.empty(torch.bfloat16, "cuda")
    sc = torch.ones(L.K, device="cuda"); bi = torch.zeros(L.K, device="cuda")
    p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
    res = []
    for bn, pair, sk in cfgs:
        if L.K % bn:
            continue
        lw = alt.Layout((L.K, L.C, L.R, L.S), LY.kcrs_yk_xc(L.K, L.C, bn, x))
        wt = lw.empty(torch.bfloat16, "cuda").normal_()
        cfg = {"path": 1, "block_n": bn, "cta_pair": pair, "split_k": sk}
        try:
            us = timeit(lambda: alt.conv2d(p, lx, xt, lw, wt, ly, yt, scale=sc, bias=bi, act="relu", cfg=cfg))
            pl = alt.last_plan()
            res.append((us, bn, pair, sk, pl["split_k"], pl["tile_n"], pl["tile_h"], pl["tile_w"]))
        except Exception as e:
            res.append((1e9, bn, pair, sk, str(e)[:40]))
    res.sort()
    print(L.name, f"{L.flops(N)/1e9:.1f} GF")
    for r in res[:8]:
        print("   ", r)
