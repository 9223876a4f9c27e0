"""store_at with the bias row contiguous: weights in the paper's K/kt N/nt kt nt
template (N innermost), Z = store_at(B, bias, 0) stored (K+kt)/kt N/nt kt nt, so
row k = K (the bias) is a contiguous nt-run per N tile.  BERT FC GEMMs at M =
8192, CUDA events, 100 launches after 10 warm-up; vs separate bias on the
same B layout and vs the tuned NK layout."""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/", 2)[0])
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY  # noqa: E402


def timed(fn, iters=100, warm=10):
    for _ in range(warm):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(iters):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / iters


dt, M = torch.bfloat16, 8192
for K, N in [(768, 768), (768, 3072), (3072, 768)]:
    La = alt.Layout((M, K), LY.gemm_a_tiled(M, K, 128, 64))
    Lc = alt.Layout((M, N), LY.gemm_c_tiled(M, N, 128, 64))
    a, c = La.empty(dt).normal_(), Lc.empty(dt)
    bias = torch.randn(N, device="cuda").to(dt)
    row = {"K": K, "N": N}
    for name, bp, zp in [("nk", LY.gemm_b_tiled_nk(K, N, 256, 64), LY.gemm_z_tiled_nk(K, N, 256, 64)),
                         ("kn", LY.gemm_b_tiled_kn(K, N, 64, 256),
                          [("pad", 0, 0, 63), ("split", 0, [(K + 64) // 64, 64]), ("split", 2, [N // 256, 256]),
                           ("reorder", [0, 2, 1, 3])])]:
        Lb, Lz = alt.Layout((K, N), bp), alt.Layout((K + 1, N), zp)
        b = Lb.empty(dt).normal_()
        z = Lz.empty(dt)
        alt.store_at(Lb, b, bias, 0, Lz, z)
        try:
            row[name + "_sep_us"] = round(timed(lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, bias=bias.float())), 2)
            row[name + "_sep_path"] = alt.last_plan()["path"]
            row[name + "_att_us"] = round(timed(lambda: alt.matmul_store_at(M, N, K, La, a, Lz, z, Lc, c)), 2)
            row[name + "_att_path"] = alt.last_plan()["path"]
        except Exception as e:  # noqa: BLE001
            row[name + "_error"] = str(e)[:120]
    print(json.dumps(row), flush=True)
