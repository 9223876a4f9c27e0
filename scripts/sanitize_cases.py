"""Small invocations of every kernel family for compute-sanitizer runs
(memcheck / racecheck / synccheck): tensor-core conv (bf16, fp32 split,
MN-major, split-K, cluster split-K, tail split, round stores, padded-output
epilogue), GEMM, depthwise, pool, relayout (permutation, K_ROW, K_CT,
generic, K_WIN, K_PBLOCK, warp-staged stores), resident weights, store_at.  Each case is checked against the oracle so a race that
corrupts data also fails here.  usage: sanitize_cases.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY  # noqa: E402
from tests.test_gpu_conv import run_conv, run_gemm  # noqa: E402
from tests.test_gpu_relayout import _gpu_relayout  # noqa: E402

BF, F32 = torch.bfloat16, torch.float32
TC = {"path": alt.PATH_TC}
cases = [
    ("tc conv 3x3 bf16", lambda: run_conv("s1", 2, 64, 14, 14, 128, 3, 3, 1, 1, LY.nchwxc(64, 64),
                                          LY.kcrs_yk_xc(128, 64, 128, 64), LY.nchwxc(128, 64), BF, epi=True, act=1, cfg=TC)),
    ("tc conv bn64 single", lambda: run_conv("s2", 2, 64, 14, 14, 64, 3, 3, 1, 1, LY.nchwxc(64, 64),
                                             LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64), BF, epi=True,
                                             res_p=LY.nchwxc(64, 64), act=1, cfg={**TC, "block_n": 64})),
    ("tc conv split-K 2", lambda: run_conv("s3", 2, 128, 7, 7, 128, 3, 3, 1, 1, LY.nchwxc(128, 64),
                                           LY.kcrs_yk_xc(128, 128, 128, 64), LY.nchwxc(128, 64), BF,
                                           cfg={**TC, "block_n": 128, "split_k": 2})),
    ("tc conv cluster split 2", lambda: run_conv("s4", 2, 128, 7, 7, 128, 3, 3, 1, 1, LY.nchwxc(128, 64),
                                                 LY.kcrs_yk_xc(128, 128, 128, 64), LY.nchwxc(128, 64), BF,
                                                 cfg={**TC, "block_n": 128, "cta_pair": 2, "split_k": 2,
                                                      "split_cluster": 1})),
    ("tc conv padded output", lambda: run_conv("s5", 2, 64, 14, 14, 64, 3, 3, 1, 1, LY.nchwxc(64, 64),
                                               LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 8, pad_hw=1), BF, cfg=TC)),
    ("tc conv fp32 split", lambda: run_conv("s6", 2, 32, 9, 9, 64, 3, 3, 1, 1, LY.nchwxc(32, 8),
                                            LY.kcrs_yk_xc(64, 32, 16, 8), LY.nhwc(), F32, epi=True, act=1, cfg=TC)),
    ("tc gemm MN-major", lambda: run_gemm("s7", 256, 128, 192, LY.transpose2(), [], [], BF, epi=True, cfg=TC)),
    ("tc gemm tail split", lambda: run_gemm("s8", 512, 768, 256, [], LY.transpose2(), [], BF,
                                            cfg={**TC, "split_k": 2, "split_cluster": 2})),
    ("depthwise", lambda: run_conv("s9", 2, 32, 14, 14, 32, 3, 3, 1, 1, LY.nchwxc(32, 8), [("reorder", [1, 2, 3, 0])],
                                   LY.nchwxc(32, 8), BF, groups=32, epi=True, act=2, cfg={"path": alt.PATH_DW})),
    ("simt conv", lambda: run_conv("s10", 1, 16, 9, 9, 24, 3, 3, 2, 1, [], [], [], F32, cfg={"path": alt.PATH_SIMT})),
    ("relayout perm", lambda: _gpu_relayout((2, 64, 14, 14), [], LY.nchwxc(64, 8), BF, "r1")),
    ("relayout pad+unfold (K_ROW)", lambda: _gpu_relayout((2, 64, 14, 14), [],
                                                         LY.conv_input_tiled(64, 8, 14, 14, 3, 3, 7, 7, 1, 1), BF, "r2")),
    ("relayout wfold (K_ROW)", lambda: _gpu_relayout((2, 3, 33, 31), [], LY.conv_input_wfold(3, 3, 2, 1), BF, "r3")),
    ("relayout generic", lambda: _gpu_relayout((2, 16, 14, 14), [("fuse", 1, 3), ("split", 1, [4, 4, 196]),
                                                                 ("reorder", [0, 1, 3, 2])], [], F32, "r4")),
    ("relayout window group (K_WIN)", lambda: _gpu_relayout((3, 16, 30, 30), [],
                                                           LY.conv_input_tiled(16, 8, 30, 30, 3, 3, 8, 8, 1, 1), BF, "r5")),
    ("relayout perm block (K_PBLOCK)", lambda: _gpu_relayout((64, 32, 3, 3), [], LY.kcrs_yk_xc(64, 32, 8, 8), BF, "r6")),
    ("relayout warp-staged rt", lambda: _gpu_relayout((3, 16, 8, 13), [], LY.nchwxc(16, 8), BF, "r7")),
    ("relayout ident fp32 32-byte runs", lambda: _gpu_relayout((2, 3, 20, 24), [], LY.nchwxc(3, 8, pad_c=5), F32, "r8")),
    ("tc conv resident weights", lambda: run_conv("s11", 8, 64, 28, 28, 64, 3, 3, 1, 1, LY.nchwxc(64, 64),
                                                  LY.kcrs_yk_xc(64, 64, 64, 64), LY.nchwxc(64, 64), BF, epi=True,
                                                  act=1, cfg={**TC, "block_n": 64})),
]
only = sys.argv[1:]
for name, fn in cases:
    if only and not any(o in name for o in only):
        continue
    fn()
    torch.cuda.synchronize()
    print("ok", name, flush=True)
