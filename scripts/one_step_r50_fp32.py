"""Build the R50 b32 LayerSet in fp32 (bench.py's aux.r50_fp32 plans) and run
warm-up + one step: the ncu target for the fp32 launch list."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
S = bench.LayerSet(32, torch.device("cuda", 0), torch.float32)
S.step()
S.step()
torch.cuda.synchronize()
