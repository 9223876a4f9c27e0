"""Halo mode vs the tuned plan on the stride-1 3x3 layers (R50 b32, R18):
time every eligible tile (W run 16 / 32 / 64 >= Wo + 2) x BLOCK_N x CTA
pair with the halo (block_k 1) and without (block_k 2), print the best of
each next to the tuned cfg.  usage: halo_probe.py [batch]"""
import itertools
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from scripts.exptime import timeit  # noqa: E402

S = bench.LayerSet(int(sys.argv[1]) if len(sys.argv) > 1 else 32, torch.device("cuda", 0))
for l in S.layers:
    L = l["L"]
    if L.R != 3 or L.stride != 1:
        continue
    Ho, Wo = L.out_hw()
    f = lambda c: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"],  # noqa: E731
                             bias=l["bi"], act="relu", cfg=c)
    tuned = timeit(lambda: f(l["cfg"]))
    best = {1: (1e9, None), 2: (1e9, None)}
    for tw in (16, 32, 64):
        if Wo + 2 > tw:
            continue
        for th in (1, 2, 4, 8):
            tn = 128 // (tw * th)
            if tn < 1 or tn * th * tw != 128:
                continue
            for bn, pr, hk in itertools.product((64, 128, 256), (0, 2), (1, 2)):
                if bn > max(64, L.K):
                    continue
                c = {"path": 1, "block_n": bn, "cta_pair": pr, "tile_n": tn, "tile_h": th, "tile_w": tw, "block_k": hk}
                try:
                    t = timeit(lambda: f(c))
                except alt.AltError:
                    continue
                if alt.last_plan()["block_k"] != (1 if hk == 1 else 64):
                    continue
                if t < best[hk][0]:
                    best[hk] = (t, c)
    print(f"{L.name:8s} tuned {tuned:6.2f} us | halo {best[1][0]:6.2f} {best[1][1]} | no-halo same tiles {best[2][0]:6.2f}",
          flush=True)
