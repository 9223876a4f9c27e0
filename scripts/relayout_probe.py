"""Time selected D6 relayout cases (developer probe for the relayout kernel
knobs).  usage: relayout_probe.py [CASE_PREFIX ...]  (default R3)"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import bench_workloads as BW  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import relayout_set  # noqa: E402

pref = sys.argv[1:] or ["R3"]
dev = torch.device("cuda", 0)
peak = bench.peaks()[1]
tag = " ".join(f"{k}={v}" for k, v in os.environ.items() if k.startswith("ALT_"))
for name, shape, sp, dp in relayout_set.cases():
    if not any(name.startswith(p) for p in pref):
        continue
    for dt in (torch.bfloat16, torch.float32):
        S, D = alt.Layout(shape, sp), alt.Layout(shape, dp)
        src = S.empty(dt, dev).normal_()
        dst = D.empty(dt, dev)
        t = BW._time(lambda: alt.relayout(S, src, D, dst), 10, 3, 1)
        nb = relayout_set.alg_bytes(S, D, src.element_size())
        print(f"{tag:40s} {name[:34]:34s} {str(dt)[6:]:9s} {t * 1e3:8.1f} us  {nb / (t * 1e-3) / 1e9 / peak:.3f}")
