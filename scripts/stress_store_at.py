"""Stress the first launch of fresh tensor-core GEMM plans with a residual
(the intermittent round-0 residual loss of test_matmul_store_at_parity):
every iteration builds new layouts / buffers (a cache-miss plan, fresh
layout tables) and checks the result against one fp64 reference.
usage: stress_store_at.py [iters] [variant]
variants: fresh (new Lc, c, z each time), newc (new c only), store (a
store_at + torch fill before each GEMM, as the test does)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from oracle.store_at import gemm_store_at_f64, store_at as o_store_at  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth  # noqa: E402

iters = int(sys.argv[1]) if len(sys.argv) > 1 else 100
variant = sys.argv[2] if len(sys.argv) > 2 else "fresh"
M, N, K, pad = 384, 192, 256, 7
dt = torch.bfloat16
A = synth.activations("msa_A", (M, K)).to(dt)
B = synth.weights("msa_B", (K, N)).to(dt)
b = synth.bn_bias("msa_b", N).to(dt)
sc = synth.bn_scale("msa_s", N)
res = synth.activations("msa_r", (M, N)).to(dt)
f64 = lambda t: t.double().numpy()  # noqa: E731
want = gemm_store_at_f64(f64(A), o_store_at(f64(B), f64(b), 0), scale=sc.double().numpy(), residual=f64(res),
                         act="relu")
tol = 0.05 * np.abs(want).max()
La, Lb = alt.Layout((M, K), []), alt.Layout((K, N), [])
zprims = [("reorder", [1, 0]), ("pad", 1, 0, pad)]
Lz = alt.Layout((K + 1, N), zprims)
z = torch.empty(Lz.phys_shape, dtype=dt, device="cuda")
alt.store_at(Lb, B.cuda(), b.cuda(), 0, Lz, z)
Lc = alt.Layout((M, N), [])
ad, rd = A.cuda(), res.cuda()
bad = 0
for it in range(iters):
    if variant in ("fresh", "store"):
        Lz = alt.Layout((K + 1, N), zprims)
        z = torch.empty(Lz.phys_shape, dtype=dt, device="cuda")
        alt.store_at(Lb, B.cuda(), b.cuda(), 0, Lz, z)
        Lc = alt.Layout((M, N), [])
        rd = res.cuda()
    c = torch.full((M, N), float("nan"), dtype=dt, device="cuda")
    alt.matmul_store_at(M, N, K, La, ad, Lz, z, Lc, c, scale=sc.cuda(), residual=rd, residual_l=Lc, act="relu",
                        cfg={"path": alt.PATH_TC})
    torch.cuda.synchronize()
    got = c.double().cpu().numpy()
    d = np.abs(got - want) > tol
    if d.any():
        bad += 1
        rows, cols = np.where(d.any(1))[0], np.where(d.any(0))[0]
        if bad <= 5:
            print(f"iter {it}: {int(d.sum())} wrong, rows {rows.min()}..{rows.max()} ({len(rows)}), "
                  f"cols {cols.min()}..{cols.max()}", flush=True)
print(f"variant {variant}: {bad} / {iters} launches wrong; plan {alt.last_plan()}", flush=True)
