"""Repeat the intermittently failing store_at TC case; print the failure rate
and where the wrong outputs are.  usage: repro_store_at.py [reps]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from oracle.store_at import gemm_store_at_f64, store_at as o_store_at  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth  # noqa: E402

M, N, K, pad = 384, 192, 256, 7
dt = torch.bfloat16
A = synth.activations("msa_A", (M, K)).to(dt)
B = synth.weights("msa_B", (K, N)).to(dt)
b = synth.bn_bias("msa_b", N).to(dt)
La, Lb = alt.Layout((M, K), []), alt.Layout((K, N), [])
Lz = alt.Layout((K + 1, N), [("reorder", [1, 0]), ("pad", 1, 0, pad)])
Lc = alt.Layout((M, N), [])
z = torch.zeros(Lz.phys_shape, dtype=dt, device="cuda")
alt.store_at(Lb, B.cuda(), b.cuda(), 0, Lz, z)
ref = gemm_store_at_f64(A.double().numpy(), o_store_at(B.double().numpy(), b.double().numpy(), 0))
ad = A.cuda()
bad = 0
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 50
for r in range(reps):
    c = torch.full((M, N), 5.0, dtype=dt, device="cuda")
    alt.matmul_store_at(M, N, K, La, ad, Lz, z, Lc, c, cfg={"path": 1})
    torch.cuda.synchronize()
    got = c.double().cpu().numpy()
    err = np.linalg.norm(got - ref) / np.linalg.norm(ref)
    if err > 2e-2:
        bad += 1
        rows = np.where(np.abs(got - ref).max(1) > 0.05 * np.abs(ref).max())[0]
        cols = np.where(np.abs(got - ref).max(0) > 0.05 * np.abs(ref).max())[0]
        print(f"rep {r}: err {err:.3e} bad rows {rows.min()}..{rows.max()} ({len(rows)}) cols {cols.min()}..{cols.max()} ({len(cols)})", flush=True)
print("plan", alt.last_plan())
print(f"{bad} / {reps} bad")
