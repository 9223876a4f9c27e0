"""Epilogue chunk timeline (ALT_TC_DEBUG=1), one tile per CTA."""
import os, sys, ctypes
os.environ["ALT_TC_DEBUG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, _alt
dt = torch.bfloat16
lib = _alt._lib
lib.alt__debug_tc.argtypes = [ctypes.c_void_p, ctypes.c_int64]
for bn, M, K, epi in [(256, 128 * 148, 64, False), (256, 128 * 148, 64, True)]:
    N = bn
    La, Lb, Lc = alt.Layout((M, K), []), alt.Layout((K, N), LY.transpose2()), alt.Layout((M, N), [])
    a, b, c = La.empty(dt).normal_(), Lb.empty(dt).normal_(), Lc.empty(dt)
    kw = dict(bias=torch.zeros(N, device="cuda"), scale=torch.ones(N, device="cuda")) if epi else {}
    for _ in range(3):
        alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg={"path": 1, "block_n": bn}, **kw)
    torch.cuda.synchronize()
    ncta = 148
    buf = np.zeros(ncta * 32, np.uint64)
    lib.alt__debug_tc(buf.ctypes.data, ncta * 32)
    t = buf.reshape(ncta, 32).astype(np.int64)
    t0 = t[:, 0].min()
    rel = (t - t0) / 1000.0
    med = np.median(rel, axis=0)
    print(f"bn={bn} epi={epi}: setup {med[1]:.2f} tfull {med[2]:.2f}")
    for ch in range(4):
        print(f"   chunk {ch}: ld {med[8+4*ch]:.2f} math {med[9+4*ch]:.2f} smem {med[10+4*ch]:.2f} store {med[11+4*ch]:.2f}")
    print(f"   epi_end {med[5]:.2f} end {med[6]:.2f}", flush=True)
