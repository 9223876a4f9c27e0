"""One epilogue-bound GEMM launch for ncu source-level profiling."""
import sys
import torch
sys.path.insert(0, ".")
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
dt = torch.bfloat16
M, K, N = 128 * 148 * 16, 64, 256
La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
sc, bi = torch.ones(N, device="cuda"), torch.zeros(N, device="cuda")
for _ in range(2):
    alt.matmul(M, N, K, La, a, Lb, b, Lc, c, scale=sc, bias=bi, act=1, cfg={"path": 1, "block_n": 256, "cta_pair": 1})
torch.cuda.synchronize()
