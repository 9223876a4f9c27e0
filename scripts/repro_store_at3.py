"""Reproduce the store_at TC failure seen after the R50 b1 set: run the b1
LayerSet once, then the 384x192x256 pad-7 store_at GEMM (NaN-poisoned
output) in several variants; report which are wrong and where."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from oracle.store_at import gemm_store_at_f64, store_at as o_store_at  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth  # noqa: E402

S = bench.LayerSet(1, torch.device("cuda", 0))
S.step()
torch.cuda.synchronize()
del S
M, N, K, pad = 384, 192, 256, 7
dt = torch.bfloat16
A = synth.activations("msa_A", (M, K)).to(dt)
B = synth.weights("msa_B", (K, N)).to(dt)
b = synth.bn_bias("msa_b", N).to(dt)
sc = synth.bn_scale("msa_s", N)
res = synth.activations("msa_r", (M, N)).to(dt)
f64 = lambda t: t.double().numpy()  # noqa: E731
for variant in ("res", "nores", "res-single", "res", "nores", "res"):
    La, Lb = alt.Layout((M, K), []), alt.Layout((K, N), [])
    Lz = alt.Layout((K + 1, N), [("reorder", [1, 0]), ("pad", 1, 0, pad)])
    Lc = alt.Layout((M, N), [])
    z = torch.empty(Lz.phys_shape, dtype=dt, device="cuda")
    alt.store_at(Lb, B.cuda(), b.cuda(), 0, Lz, z)
    c = torch.full((M, N), float("nan"), dtype=dt, device="cuda")
    kw = dict(residual=res.cuda(), residual_l=Lc) if variant.startswith("res") else {}
    cfg = {"path": 1, "cta_pair": 2, "block_n": 128} if variant == "res-single" else {"path": 1}
    alt.matmul_store_at(M, N, K, La, A.cuda(), Lz, z, Lc, c, scale=sc.cuda(), act="relu", cfg=cfg, **kw)
    torch.cuda.synchronize()
    want = gemm_store_at_f64(f64(A), o_store_at(f64(B), f64(b), 0), scale=sc.double().numpy(),
                             residual=f64(res) if kw else None, act="relu")
    got = c.double().cpu().numpy()
    err = np.linalg.norm(got - want) / np.linalg.norm(want)
    d = np.abs(got - want) > 0.05 * np.abs(want).max()
    rows, cols = np.where(d.any(1))[0], np.where(d.any(0))[0]
    print(variant, f"err {err:.3e}", alt.last_plan()["cta_pair"], "bad rows", len(rows),
          (rows.min(), rows.max()) if len(rows) else "", "cols", (cols.min(), cols.max()) if len(cols) else "",
          "nan", int(np.isnan(got).sum()), flush=True)
