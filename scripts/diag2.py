"""GEMM vs conv of the same GEMM shape: is the conv A-box or the epilogue the limit?"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from scripts.exptime import timeit
dt = torch.bfloat16
M = 100352
for N, K in [(64, 576), (64, 64), (64, 128), (64, 256), (128, 576), (256, 576), (128, 64), (256, 64)]:
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).uniform_(-1, 1), Lb.empty(dt).uniform_(-1, 1), Lc.empty(dt)
    for pair in (1, 2):
        for st in (0,):
            try:
                us = timeit(lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": N, "cta_pair": pair}))
            except Exception as e:
                continue
            byt = 2 * (M * K + M * N)
            print(f"GEMM {M}x{N}x{K} pair={pair}: {us:.1f} us {2*M*N*K/us/1e6:.0f} TFLOP/s {byt/us/1e3:.0f} GB/s", alt.last_plan()['stages'], flush=True)
    bt = b.view(N, K).t()
    us = timeit(lambda: torch.matmul(a.view(M, K), bt))
    print(f"  cuBLAS {us:.1f} us {2*M*N*K/us/1e6:.0f} TFLOP/s", flush=True)
