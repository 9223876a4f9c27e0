"""Output-layout probe: one ResNet-50 b32 layer (bench.py's x / w layouts and
kernel cfg) timed with y = NCHW[x]c for x = 16 / 32 / 64 / 128 / 256 (one TMA
store box per x-channel slab and round: fewer, larger store requests as x
grows).  usage: store_box_probe.py LAYER[,LAYER]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY  # noqa: E402
from scripts.exptime import timeit  # noqa: E402

S = bench.LayerSet(32, torch.device("cuda", 0))
for name in sys.argv[1].split(","):
    l = [l for l in S.layers if l["L"].name == name][0]
    L = l["L"]
    Ho, Wo = L.out_hw()
    out = []
    for xc in (16, 32, 64, 128, 256):
        if L.K % xc:
            continue
        ly = alt.Layout((32, L.K, Ho, Wo), LY.nchwxc(L.K, xc))
        y = ly.empty(torch.bfloat16, torch.device("cuda", 0))
        f = lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], ly, y, scale=l["sc"],  # noqa: E731
                               bias=l["bi"], act="relu", cfg=l["cfg"])
        t = timeit(f)
        out.append(f"{xc}c:{t:.1f}")
    print(name, " ".join(out), flush=True)
