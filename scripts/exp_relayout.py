import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import relayout_set
from scripts.exptime import timeit
for dt in (torch.bfloat16, torch.float32):
    for name, shape, sp, dp in relayout_set.cases():
        S, D = alt.Layout(shape, sp), alt.Layout(shape, dp)
        src = S.empty(dt).normal_()
        dst = D.empty(dt)
        us = timeit(lambda: alt.relayout(S, src, D, dst), reps=10)
        b = relayout_set.alg_bytes(S, D, src.element_size())
        print(f"{str(dt)[6:]:9s} {name:40s} {us:8.1f} us  {b/us/1e3:7.0f} GB/s  ({b/1e6:.0f} MB)", flush=True)
