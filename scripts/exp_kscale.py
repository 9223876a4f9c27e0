"""Per-iteration cost of the TC kernel: one full wave of CTAs (148 M tiles),
K swept, stages swept."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from scripts.exptime import timeit
dt = torch.bfloat16
for bn, st in [(128, 2), (128, 4), (128, 6), (256, 2), (256, 4)]:
    for M, kk in [(128 * 148, 1), (128 * 148, 4), (128 * 148, 16), (128 * 148, 64), (128 * 148 * 4, 64)]:
        K = 64 * kk
        N = bn
        La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
        a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
        f = lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "stages": st})
        us = timeit(f)
        print(f"bn={bn} stages={st} M={M} K={K}: {us:.1f} us  {2*M*N*K/us/1e6:.1f} TF/s  plan={alt.last_plan()['stages']}", flush=True)
