"""alt_tune over the ResNet-50 layer set (BASELINE config 2) at a batch:
stores every winner in tune_cache.jsonl (the bench's layouts + kernel cfgs).
Few-channel layers (conv1, C % 8 != 0) keep the window-folded template.
usage: tune_r50.py [N] [OUT_COPY]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets, tunecache

N = int(sys.argv[1]) if len(sys.argv) > 1 else 32
def tune_folded(L, N):
    """few-channel layers (conv1): the window-folded template is fixed
    (reading A23); only the loop schedule (output-pixel tile) is measured."""
    import torch
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
    from scripts.exptime import timeit
    Ho, Wo = L.out_hw()
    xp, wp, yp = LY.conv_input_wfold(L.C, L.S, L.stride, L.pad), LY.kcrs_wfold(L.K, L.C, L.S), LY.nchwxc(L.K, 64)
    lx, lw, ly = (alt.Layout((N, L.C, L.H, L.W), xp), alt.Layout((L.K, L.C, L.R, L.S), wp),
                  alt.Layout((N, L.K, Ho, Wo), yp))
    xt, wt, yt = lx.empty(torch.bfloat16).normal_(), lw.empty(torch.bfloat16).normal_(), ly.empty(torch.bfloat16)
    sc, bi = torch.ones(L.K, device="cuda"), torch.zeros(L.K, device="cuda")
    p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
    best = None
    for th in (1, 2, 4, 8, 16):
        for tw in (8, 16, 32, 64):
            tn = 128 // (th * tw)
            if tn < 1 or tn > N:
                continue
            cfg = {"path": 1, "block_n": 64, "cta_pair": 2, "tile_n": tn, "tile_h": th, "tile_w": tw}
            us = timeit(lambda: alt.conv2d(p, lx, xt, lw, wt, ly, yt, scale=sc, bias=bi, act="relu", cfg=cfg))
            if best is None or us < best[0]:
                best = (us, cfg)
    tunecache.store("conv2d", L, N, {"x": xp, "w": wp, "y": yp, "cfg": best[1], "best_us": best[0]})
    print(f"{L.name:10s} best {best[0]:7.2f} us (window-folded, tile sweep) cfg={best[1]}", flush=True)


for L in nets.RESNET50:
    if L.C % 8:
        tune_folded(L, N)
        continue
    p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
    Ho, Wo = L.out_hw()
    tws = [0] + [t for t in (4, 8, 16, 32) if t <= 2 * Wo]
    space = {0: [64, 32], 1: [64, 32], 2: [1, 2, 4, -2, -4], 3: [0, 2], 4: [1, 2, 4], 5: tws, 6: [256, 128, 64],
             7: [0, 1] if L.R > 1 else [0]}
    t0 = time.time()
    r = alt.tune("conv2d", p, alt.ALT_BF16, space, max_points=4096, warmup=3, reps=10)
    tunecache.store("conv2d", L, N, r)
    print(f"{L.name:10s} best {r['best_us']:7.2f} us of {r['measured']} points ({time.time() - t0:.1f} s) "
          f"cfg={ {k: r['cfg'][k] for k in ('block_n', 'cta_pair', 'tile_n', 'tile_h', 'tile_w')} } "
          f"x={r['x'][-2:]}", flush=True)
if len(sys.argv) > 2:
    import shutil
    shutil.copy(tunecache._PATH, sys.argv[2])
