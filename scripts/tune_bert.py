"""Kernel-configuration sweep for the BERT-base GEMMs (BASELINE config 3, M = 8192)
on the bench's tiled layouts; winners go to tune_cache.jsonl (key matmul|M|N|K)."""
import itertools, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, nets, tunecache
from scripts.exptime import timeit
M = 8192
for name, K, N in nets.BERT_GEMMS:
    La = alt.Layout((M, K), LY.gemm_a_tiled(M, K, 128, 64))
    Lc = alt.Layout((M, N), LY.gemm_c_tiled(M, N, 128, 64))
    a, c = La.empty(torch.bfloat16).normal_(), Lc.empty(torch.bfloat16)
    res = []
    # joint layout + loop point: the B tile nt of the layout N/nt K/64 nt 64 and the kernel's BLOCK_N
    for nt in (256, 192):
        if N % nt:
            continue
        Lb = alt.Layout((K, N), LY.gemm_b_tiled_nk(K, N, nt, 64))
        b = Lb.empty(torch.bfloat16).normal_()
        bns = (128, 256) if nt == 256 else (192,)
        for bn, pair, sk, scl in itertools.product(bns, (0, 2), (1, 2, 3, 4), (0, 1, 2)):
            if scl == 1 and (pair != 2 or sk == 1 or sk == 3):
                continue
            if scl == 2 and sk == 1:
                continue
            cfg = {"path": 1, "block_n": bn, "cta_pair": pair, "split_k": sk, "split_cluster": scl}
            try:
                us = timeit(lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg=cfg))
                res.append((us, dict(cfg, b_nt=nt)))
            except alt.AltError:
                pass
    res.sort(key=lambda r: r[0])
    best_us, best = res[0]
    tunecache.store_gemm(M, N, K, best, best_us)
    print(f"{name}: best {best_us:.2f} us {2 * M * N * K / best_us / 1e6:.0f} TFLOP/s {best}; "
          f"runner-up {[(round(u, 2), c['b_nt'], c['block_n'], c['cta_pair'], c['split_k'], c['split_cluster']) for u, c in res[1:4]]}",
          flush=True)
if len(sys.argv) > 1:
    import shutil
    shutil.copy(tunecache._PATH, sys.argv[1])
