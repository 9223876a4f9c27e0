"""Per-layer device time of the R50 b32 set (graph of repeated launches),
for the epilogue A/B: run under ALT_TC_EPI_DBG=0 (normal), 1 (no output
stores) and 2 (no TMEM drain at all).  usage: epi_probe.py [layers]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from scripts.exptime import timeit  # noqa: E402

S = bench.LayerSet(int(os.environ.get("BATCH", "32")), torch.device("cuda", 0))
names = sys.argv[1].split(",") if len(sys.argv) > 1 else [l["L"].name for l in S.layers]
tot = 0.0
for l in S.layers:
    if l["L"].name not in names:
        continue
    f = lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"], bias=l["bi"],  # noqa: E731
                           act="relu", cfg=l["cfg"])
    t = timeit(f)
    tot += t
    print(f"{l['L'].name:10s} {t:7.2f} us  {alt.last_plan()}", flush=True)
print(f"total {tot:.1f} us")
