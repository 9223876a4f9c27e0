"""Run one ResNet-50 layer (bench.py's layout plan) a few times: ncu target."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets
names = sys.argv[1].split(",")
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
N = int(sys.argv[3]) if len(sys.argv) > 3 else 32
dev = torch.device("cuda", 0)
S = bench.LayerSet(N, dev)
S.layers = [l for l in S.layers if l["L"].name in names]
for _ in range(reps):
    S.step()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    S.step()
e1.record(); torch.cuda.synchronize()
print("us per step", e0.elapsed_time(e1) / 10 * 1e3)
