"""Time the BERT-base GEMMs (M = 8192, bench layouts) for a few kernel
configurations under the current environment (developer probe; combine with
ALT_TC_EPI_DBG=2 / 3 to strip the drain / the MMAs).  usage: gemm_probe.py"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY, nets  # noqa: E402
from scripts.exptime import timeit  # noqa: E402

M = 8192
tag = os.environ.get("ALT_TC_EPI_DBG", "0")
for name, K, N in nets.BERT_GEMMS:
    La = alt.Layout((M, K), LY.gemm_a_tiled(M, K, 128, 64))
    Lc = alt.Layout((M, N), LY.gemm_c_tiled(M, N, 128, 64))
    Lb = alt.Layout((K, N), LY.gemm_b_tiled_nk(K, N, 256, 64))
    a, b, c = La.empty(torch.bfloat16).normal_(), Lb.empty(torch.bfloat16).normal_(), Lc.empty(torch.bfloat16)
    out = []
    for bn, pair in ((256, 2), (256, 1), (128, 1), (128, 2)):
        cfg = {"path": 1, "block_n": bn, "cta_pair": pair, "split_k": 1, "split_cluster": 0}
        us = timeit(lambda: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg=cfg))
        st = alt.last_plan()["stages"]
        out.append(f"bn{bn}{'pair' if pair == 1 else 'single'}(st{st}) {us:6.1f} us {2 * M * N * K / us / 1e6:5.0f} TF")
    print(f"dbg{tag} {name:16s} " + "  ".join(out), flush=True)
