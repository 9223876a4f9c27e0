"""Per-CTA timeline of the TC kernel (ALT_TC_DEBUG=1)."""
import os, sys, ctypes
os.environ["ALT_TC_DEBUG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, _alt
dt = torch.bfloat16
lib = _alt._lib
lib.alt__debug_tc.argtypes = [ctypes.c_void_p, ctypes.c_int64]
for bn, M, K in [(128, 128 * 148, 64), (256, 128 * 148, 64), (256, 128 * 148 * 5, 64), (128, 128 * 148, 4096), (256, 128*148, 4096)]:
    N = bn
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
    for _ in range(3):
        alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn})
    torch.cuda.synchronize()
    ncta = min(148, (M // 128) * (N // bn))
    buf = np.zeros(ncta * 8, np.uint64)
    lib.alt__debug_tc(buf.ctypes.data, ncta * 8)
    t = buf.reshape(ncta, 8).astype(np.int64)
    t0 = t[:, 0].min()
    rel = (t - t0) / 1000.0
    names = ["start", "setup", "epi_tfull0", "mma_tile0_done", "-", "epi_end", "end"]
    print(f"bn={bn} M={M} K={K}: medians (us from first CTA start):",
          {n: round(float(np.median(rel[:, i])), 2) for i, n in enumerate(names)},
          "max end", round(float(rel[:, 6].max()), 2), "start spread", round(float(rel[:, 0].max()), 2), flush=True)
