#!/bin/bash
cd $GRAFT_REPO_ROOT
true
python - <<'PY' 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
import sys; sys.path.insert(0, ".")
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, nets
from scripts.exptime import timeit
N = 32
for L in nets.RESNET50:
    if L.name not in ("l4.3x3", "l4.3x3s2", "l3.3x3", "l4.1x1c", "l4.1x1b", "l3.3x3s2", "l4.1x1a", "l3.1x1b"): continue
    Ho, Wo = L.out_hw()
    xp, yp = LY.nchwxc(L.C, 64), LY.nchwxc(L.K, 64)
    lx, ly = alt.Layout((N, L.C, L.H, L.W), xp), alt.Layout((N, L.K, Ho, Wo), yp)
    xt = lx.empty(torch.bfloat16, "cuda").normal_(); yt = ly.empty(torch.bfloat16, "cuda")
    sc = torch.ones(L.K, device="cuda"); bi = torch.zeros(L.K, device="cuda")
    p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
    res = []
    for bn in (128, 256):
        lw = alt.Layout((L.K, L.C, L.R, L.S), LY.kcrs_yk_xc(L.K, L.C, bn, 64))
        wt = lw.empty(torch.bfloat16, "cuda").normal_()
        for sk, scl in ((1, 0), (2, 1), (4, 1)):
            for tiles in (None, (16, 1, 8), (32, 2, 2), (8, 2, 8)):
                cfg = {"path": 1, "block_n": bn, "cta_pair": 2, "split_k": sk, "split_cluster": scl}
                if tiles: cfg.update(tile_n=tiles[0], tile_h=tiles[1], tile_w=tiles[2])
                try:
                    us = timeit(lambda: alt.conv2d(p, lx, xt, lw, wt, ly, yt, scale=sc, bias=bi, act="relu", cfg=cfg))
                    res.append((round(us, 2), bn, sk, scl, tiles))
                except Exception as e:
                    res.append((1e9, bn, sk, scl, tiles, str(e)[:50]))
    res.sort(key=lambda r: r[0])
    print(L.name, res[:6], flush=True)
PY
