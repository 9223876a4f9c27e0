"""Steady-state epilogue throughput: GEMM with one k-iteration per tile,
many tiles per CTA.  Reports us per tile per CTA and output GB/s."""
import sys
import torch
sys.path.insert(0, ".")
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from scripts.exptime import timeit
dt = torch.bfloat16
import os
for K in [int(k) for k in os.environ.get('EPI_K', '64,256').split(',')]:
    for bn, pair in ((64, 2), (128, 2), (256, 2)):
        for tiles_per_cta in (32,):
            M = 128 * 148 * tiles_per_cta // (1 if pair == 2 else 1)
            N = bn * 1
            La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
            a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
            sc, bi = torch.ones(N, device="cuda"), torch.zeros(N, device="cuda")
            us = timeit(lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, scale=sc, bias=bi, act=1,
                                           cfg={"path": 1, "block_n": bn, "cta_pair": pair}))
            out = M * N * 2
            inp = M * K * 2
            print(f"K={K} bn={bn} pair={pair} tiles/cta={tiles_per_cta}: {us:.1f} us, {us / tiles_per_cta:.2f} us/tile,"
                  f" out {out / us / 1e3:.0f} GB/s, in+out {(out + inp) / us / 1e3:.0f} GB/s", flush=True)
