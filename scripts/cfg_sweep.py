"""Per-layer kernel-config sweep (graph-timed): block_n x cta_pair x split_k."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from scripts.exptime import timeit
names = sys.argv[1].split(",") if len(sys.argv) > 1 else None
S = bench.LayerSet(32, torch.device("cuda", 0))
for l in S.layers:
    if names and l["L"].name not in names:
        continue
    res = []
    for bn in (64, 128, 256):
        if l["L"].K % bn and bn != 64:
            continue
        for pair in (1, 2):
            if pair == 1 and bn < 128:
                continue
            for sk in (1, 2, 4):
                cfg = dict(l["cfg"]); cfg.update(block_n=bn, cta_pair=pair, split_k=sk)
                try:
                    us = timeit(lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"], bias=l["bi"], act="relu", cfg=cfg))
                except Exception as e:
                    continue
                res.append((us, bn, pair, sk))
    res.sort()
    print(l["L"].name, " ".join(f"{us:.1f}us(bn{bn},{'pair' if p==1 else 'cta'},sk{sk})" for us, bn, p, sk in res[:6]), flush=True)
