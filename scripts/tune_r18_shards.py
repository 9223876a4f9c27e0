"""Tune the R18 chain at the per-GPU batches of the 2/4/8-GPU shards (chain_tune.json)
and time each shard chain (CUDA graph), to see the scaling headroom on one GPU."""
import os, sys, shutil
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
import bench_workloads as BW
dev = torch.device("cuda", 0)
for N in (256, 128, 64, 32):
    ch = CH.resnet18(N, dev)
    if N != 256:
        ch.tune()
    ms = BW._time(lambda: ch.run(), 10, 3, 1)
    print(f"r18 per-GPU batch {N}: {ms:.3f} ms/step, {ch.flops / (ms * 1e-3) / 1e12:.1f} TFLOP/s; ideal 8-GPU scaling from b256 needs <= {1.8 / 8:.3f} ms at b32", flush=True)
    del ch
    torch.cuda.empty_cache()
shutil.copy(CH._TUNE_PATH, sys.argv[1])
