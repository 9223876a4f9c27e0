"""Steady-state epilogue chunk timeline (build with EXTRA=-DALT_DBG_TILE=4, ALT_TC_DEBUG=1)."""
import os, sys, ctypes
os.environ["ALT_TC_DEBUG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, _alt
dt = torch.bfloat16
lib = _alt._lib
lib.alt__debug_tc.argtypes = [ctypes.c_void_p, ctypes.c_int64]
for bn, pair, K, cl in [(256, 2, 64, []), (64, 2, 64, []), (256, 2, 64, LY.gemm_c_tiled(128 * 148 * 16, 256, 128, 64))]:
    M = 128 * 148 * 16
    N = bn
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), cl)
    a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
    kw = dict(bias=torch.zeros(N, device="cuda"), scale=torch.ones(N, device="cuda"))
    for _ in range(3):
        alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn, "cta_pair": pair}, **kw)
    torch.cuda.synchronize()
    ncta = 148
    buf = np.zeros(ncta * 32, np.uint64)
    lib.alt__debug_tc(buf.ctypes.data, ncta * 32)
    t = buf.reshape(ncta, 32).astype(np.int64)
    rel = (t - t[:, 2:3]) / 1000.0  # relative to tfull of the followed tile
    med = np.median(rel, axis=0)
    print(f"bn={bn} pair={pair} out={'tiled' if cl else 'rowmajor'}: start->tfull {-med[0]:.2f} us")
    for ch in range(bn // 64):
        print(f"   chunk {ch}: ld {med[8+4*ch]:.3f} math {med[9+4*ch]:.3f} smem {med[10+4*ch]:.3f} store {med[11+4*ch]:.3f}")
    print(f"   epi_end {med[5]:.2f} end {med[6]:.2f}", flush=True)
