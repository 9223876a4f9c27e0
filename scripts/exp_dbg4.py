"""Steady-state per-role timeline of one tile (build EXTRA=-DALT_DBG_TILE=8, ALT_TC_DEBUG=1)."""
import os, sys, ctypes
os.environ["ALT_TC_DEBUG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, _alt
dt = torch.bfloat16
lib = _alt._lib
lib.alt__debug_tc.argtypes = [ctypes.c_void_p, ctypes.c_int64]
names = {24: "prod: before empty wait", 25: "prod: after empty wait", 26: "mma: before tempty", 27: "mma: after tempty",
         28: "mma: first full", 29: "mma: commit tfull", 2: "epi: tfull", 30: "epi: sb staged", 8: "epi: c0 ld",
         9: "epi: c0 math", 10: "epi: c0 smem", 11: "epi: c0 store", 12: "epi: c1 ld", 15: "epi: c1 store", 31: "epi: tile end"}
for bn, pair, K in [(64, 2, 64), (128, 1, 64), (64, 2, 256), (256, 2, 64)]:
    M = 128 * 148 * 32
    N = bn
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
    kw = dict(bias=torch.zeros(N, device="cuda"), scale=torch.ones(N, device="cuda"))
    for _ in range(3):
        alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "cta_pair": pair}, **kw)
    torch.cuda.synchronize()
    ncta = 148
    buf = np.zeros(ncta * 32, np.uint64)
    lib.alt__debug_tc(buf.ctypes.data, ncta * 32)
    t = buf.reshape(ncta, 32).astype(np.int64)
    rel = (t - t[:, 2:3]) / 1000.0
    med = np.median(rel, axis=0)
    print(f"bn={bn} pair={pair} K={K}: (us relative to epilogue tfull of tile 8)")
    for k in sorted(names, key=lambda k: med[k]):
        print(f"   {names[k]:26s} {med[k]:8.3f}")
    print(f"   kernel total {(np.median(t[:, 6]) - np.median(t[:, 0])) / 1000:.1f} us", flush=True)
