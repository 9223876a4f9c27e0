"""Loop-tune the R18 chain (chain.tune: BLOCK_N, CTA pair, split-K, pixel
tiles, halo tiles) at the per-GPU batches of the 1/2/4/8-GPU shards of the
global batch 256 (chain_tune.json) and time each shard chain before / after
(CUDA graph).  usage: tune_r18_shards.py OUT_COPY [N ...]"""
import os
import shutil
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench_workloads as BW  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH  # noqa: E402

dev = torch.device("cuda", 0)
for N in ([int(v) for v in sys.argv[2:]] or (256, 128, 64, 32)):
    ch = CH.resnet18(N, dev)
    before = BW._time(lambda: ch.run(), 10, 3, 1)
    ch.tune(log=lambda m: print(f"r18 N{N}", m, flush=True))
    after = BW._time(lambda: ch.run(), 10, 3, 1)
    print(f"r18 per-GPU batch {N}: {before:.3f} -> {after:.3f} ms/step, {ch.flops / (after * 1e-3) / 1e12:.1f} TFLOP/s",
          flush=True)
    del ch
    torch.cuda.empty_cache()
    shutil.copy(CH._TUNE_PATH, sys.argv[1])
