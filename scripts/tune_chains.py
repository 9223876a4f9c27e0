"""Loop tuning of the R18 / MV2 chains with propagated layouts (chain.tune);
writes chain_tune.json.  usage: tune_chains.py OUT_COPY"""
import os, sys, shutil
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
dev = torch.device("cuda", 0)
for name, N in (("mv2", 16), ("r18", 256), ("mv2", 1)):
    ch = CH.resnet18(N, dev) if name == "r18" else CH.mobilenet_v2(N, dev)
    ch.tune(log=lambda m: print(name, N, m, flush=True))
    del ch
    torch.cuda.empty_cache()
shutil.copy(CH._TUNE_PATH, sys.argv[1])
