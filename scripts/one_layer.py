"""Run one ResNet-50 layer (bench.py's plan) with a cfg override: ncu target.
usage: one_layer.py NAME [split_k] [reps] [block_n] [cta_pair]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from scripts.exptime import timeit
name = sys.argv[1]
sk = int(sys.argv[2]) if len(sys.argv) > 2 else 1
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
S = bench.LayerSet(32, torch.device("cuda", 0))
l = [l for l in S.layers if l["L"].name == name][0]
cfg = dict(l["cfg"]); cfg["split_k"] = sk
if len(sys.argv) > 4: cfg["block_n"] = int(sys.argv[4])
if len(sys.argv) > 5: cfg["cta_pair"] = int(sys.argv[5])
f = lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"], bias=l["bi"], act="relu", cfg=cfg)
for _ in range(reps):
    f()
torch.cuda.synchronize()
print(name, cfg, alt.last_plan(), f"{timeit(f):.1f} us")
