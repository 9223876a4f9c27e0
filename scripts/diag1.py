"""Mainloop ceiling: plain GEMMs (row-major A, K-major B) and split-K on one layer."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from scripts.exptime import timeit
dt = torch.bfloat16
for (M, N, K) in [(8192, 768, 3072), (8192, 768, 768), (512, 3072, 768)]:
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).uniform_(-1, 1), Lb.empty(dt).uniform_(-1, 1), Lc.empty(dt)
    for bn, pair in ((128, 1), (256, 1), (128, 2), (256, 2)):
        try:
            us = timeit(lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "cta_pair": pair}))
        except Exception as e:
            print(M, N, K, bn, pair, "ERR", e); continue
        print(f"GEMM {M}x{N}x{K} bn={bn} pair={pair}: {us:.1f} us {2*M*N*K/us/1e6:.0f} TFLOP/s", flush=True)
    bt = b.view(N, K).t()
    us = timeit(lambda: torch.matmul(a.view(M, K), bt))
    print(f"  cuBLAS {us:.1f} us {2*M*N*K/us/1e6:.0f} TFLOP/s", flush=True)
import bench
S = bench.LayerSet(32, torch.device("cuda", 0))
for l in S.layers:
    if l["L"].name not in ("l4.3x3", "l3.3x3", "l1.1x1a", "l1.3x3", "conv1"):
        continue
    for sk in (1, 2, 3, 4, 6):
        cfg = dict(l["cfg"]); cfg["split_k"] = sk
        us = timeit(lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"], bias=l["bi"], act="relu", cfg=cfg))
        print(f"{l['L'].name} split {sk}: {us:.1f} us {l['L'].flops(32)/us/1e6:.0f} TFLOP/s", alt.last_plan(), flush=True)
    # cuDNN reference for context
    import torch.nn.functional as F
    L = l["L"]
    xx = torch.randn(32, L.C, L.H, L.W, device="cuda", dtype=dt).to(memory_format=torch.channels_last)
    ww = torch.randn(L.K, L.C, L.R, L.S, device="cuda", dtype=dt).to(memory_format=torch.channels_last)
    us = timeit(lambda: F.conv2d(xx, ww, stride=L.stride, padding=L.pad))
    print(f"  cuDNN {L.name}: {us:.1f} us {L.flops(32)/us/1e6:.0f} TFLOP/s", flush=True)
