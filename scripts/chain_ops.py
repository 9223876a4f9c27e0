"""Per-op device time of a chain (eager, CUDA events around each op).
usage: chain_ops.py r18|mv2 N"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import _alt as A
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
which, N = sys.argv[1], int(sys.argv[2])
dev = torch.device("cuda", 0)
ch = CH.resnet18(N, dev) if which == "r18" else CH.mobilenet_v2(N, dev)
for _ in range(3): ch.run()
torch.cuda.synchronize()
# wrap the C-ABI calls to record events
rec = []
orig = {n: getattr(A, n) for n in ("relayout", "conv2d", "pool2d")}
def wrap(n):
    def f(*a, **k):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); r = orig[n](*a, **k); e1.record()
        desc = n
        if n == "conv2d":
            p = a[0]; desc = f"conv C{p.C} K{p.K} {p.H}x{p.W} r{p.R} s{p.stride_h} g{p.groups} plan={A.last_plan()}"
        rec.append((desc, e0, e1)); return r
    return f
for n in orig: setattr(A, n, wrap(n))
for rep in range(3):
    rec.clear(); ch.run()
torch.cuda.synchronize()
tot = 0
rows = []
for d, e0, e1 in rec:
    t = e0.elapsed_time(e1) * 1e3; tot += t; rows.append((t, d))
for t, d in rows: print(f"{t:8.1f} us  {d}")
print(f"total {tot:.1f} us over {len(rows)} ops")
