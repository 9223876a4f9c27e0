"""Epilogue cost per tile: GEMMs with many tiles per SM and short K."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from scripts.exptime import timeit
dt = torch.bfloat16
for (N, K, bn, pair) in [(64, 64, 64, 2), (128, 64, 128, 2), (256, 64, 256, 2), (256, 512, 256, 2), (256, 64, 256, 1)]:
    for tps in (2, 10):
        M = 128 * 148 * tps
        La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
        a, b, c = La.empty(dt).uniform_(-1, 1), Lb.empty(dt).uniform_(-1, 1), Lc.empty(dt)
        f = lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "cta_pair": pair})
        us = timeit(f)
        print(f"N={N} K={K} bn={bn} pair={pair} tiles/SM={tps}: {us:.2f} us", flush=True)
