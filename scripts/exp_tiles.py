"""Timing experiments for the tensor-core kernel: one layer under several
configs, plus GEMMs of the same size (2-D boxes)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY

def timeit(fn, reps=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3

dt = torch.bfloat16
def conv_case(N, C, H, K, R, s, x, cfg):
    Ho = (H + 2 * (R // 2) - R) // s + 1
    Lx = alt.Layout((N, C, H, H), LY.nchwxc(C, x)); Lw = alt.Layout((K, C, R, R), LY.kcrs_yk_xc(K, C, min(K, 256), x))
    Ly = alt.Layout((N, K, Ho, Ho), LY.nchwxc(K, min(K, 64)))
    xt, wt, yt = Lx.empty(dt).normal_(), Lw.empty(dt).normal_(), Ly.empty(dt)
    p = alt.conv_params(N, C, H, H, K, R, R, s, R // 2)
    f = lambda: alt.conv2d(p, Lx, xt, Lw, wt, Ly, yt, cfg=cfg)
    us = timeit(f)
    fl = 2 * N * K * Ho * Ho * C * R * R
    return us, fl / us / 1e6, alt.last_plan()

def gemm_case(M, N, K, bn):
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
    f = lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn})
    us = timeit(f)
    return us, 2 * M * N * K / us / 1e6, alt.last_plan()

out = []
for M, N, K in [(25088, 128, 1152), (8192, 3072, 768), (8192, 768, 3072), (16384, 4096, 4096)]:
    for bn in (128, 256):
        if N % bn: continue
        us, tf, pl = gemm_case(M, N, K, bn)
        print(f"gemm {M}x{N}x{K} bn={bn}: {us:.1f} us {tf:.1f} TF/s", flush=True)
for cfg in [{"path": 1}, {"path": 1, "tile_n": 32, "tile_h": 1, "tile_w": 4}, {"path": 1, "tile_n": 2, "tile_h": 4, "tile_w": 16},
            {"path": 1, "tile_n": 1, "tile_h": 8, "tile_w": 16}, {"path": 1, "tile_n": 4, "tile_h": 4, "tile_w": 8}]:
    for bn in (128,):
        c = dict(cfg); c["block_n"] = bn
        us, tf, pl = conv_case(32, 128, 28, 128, 3, 1, 64, c)
        print(f"conv l2.3x3 {c}: {us:.1f} us {tf:.1f} TF/s plan {pl}", flush=True)
