import sys, torch
sys.path.insert(0, '.')
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from tests.test_gpu_conv import run_conv
for C in (64, 128, 256, 512):
    for sk in (1, 2, 4):
        err, plan = run_conv("f32e", 8, C, 14, 14, 256, 3, 3, 1, 1, LY.nchwxc(C, 64), LY.kcrs_yk_xc(256, C, 256, 64),
                             LY.nchwxc(256, 64), torch.float32, epi=False, act=0, cfg={"path": 1, "split_k": sk}) if False else (None, None)
        try:
            err, plan = run_conv("f32e", 8, C, 14, 14, 256, 3, 3, 1, 1, LY.nchwxc(C, 64), LY.kcrs_yk_xc(256, C, 256, 64),
                                 LY.nchwxc(256, 64), torch.float32, cfg={"path": 1, "split_k": sk})
        except AssertionError as e:
            err = str(e)
        print("C", C, "K", C * 9, "split", sk, err, flush=True)
