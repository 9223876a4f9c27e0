"""One HBM-bound GEMM (K = 64, BN = 256, CTA pairs, 10 tiles per SM) for an ncu capture of the epilogue."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
dt = torch.bfloat16
N, K, bn = 256, 64, 256
M = 128 * 148 * 10
La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
a, b, c = La.empty(dt).uniform_(-1, 1), Lb.empty(dt).uniform_(-1, 1), Lc.empty(dt)
for _ in range(3):
    alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "cta_pair": 1})
torch.cuda.synchronize()
