"""Time chosen R50 layers with the smem ring limited to s stages (cfg
stages), for s = 2 .. deepest: is the operand pipeline latency-bound (time
falls with depth) or rate-bound (flat)?  Run under ALT_TC_EPI_DBG=3 for the
TMA pipeline alone.  usage: stage_probe.py layer,layer"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from scripts.exptime import timeit  # noqa: E402

S = bench.LayerSet(32, torch.device("cuda", 0))
for name in sys.argv[1].split(","):
    l = [l for l in S.layers if l["L"].name == name][0]
    out = []
    for st in (2, 3, 4, 5, 6, 7):
        cfg = dict(l["cfg"], stages=st)
        f = lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"],  # noqa: E731
                               bias=l["bi"], act="relu", cfg=cfg)
        t = timeit(f)
        out.append(f"{alt.last_plan()['stages']}:{t:.1f}")
    print(name, " ".join(out), flush=True)
