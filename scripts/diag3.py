"""Fixed per-launch cost: tiny GEMMs in a CUDA graph (PDL on / off)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from scripts.exptime import timeit
dt = torch.bfloat16
for (M, N, K, bn, pair) in [(128, 64, 64, 64, 2), (128 * 148, 64, 64, 64, 2), (128 * 148, 256, 64, 256, 2), (128*148, 256, 512, 256, 2),
                            (128 * 148 * 4, 64, 64, 64, 2), (128 * 148 * 4, 256, 64, 256, 2), (128*148*4, 256, 512, 256, 2)]:
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).uniform_(-1, 1), Lb.empty(dt).uniform_(-1, 1), Lc.empty(dt)
    f = lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "cta_pair": pair})
    us = timeit(f)
    us1 = timeit(f, graph=False)
    print(f"GEMM M={M} N={N} K={K} bn={bn}: graph {us:.2f} us/call, eager {us1:.2f}; tiles/SM {M*N/128/bn/148:.1f}", flush=True)
