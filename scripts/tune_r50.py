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
for L in nets.RESNET50:
    if L.C % 8:
        continue
    p = alt.conv_params(N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad)
    Ho, Wo = L.out_hw()
    tws = [0] + [t for t in (4, 8, 16, 32) if t <= 2 * Wo]
    space = {0: [64, 32], 1: [64], 2: [1, 2, 4, -2, -4], 3: [0, 2], 4: [1, 2, 4], 5: tws, 6: [256, 128, 64],
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
