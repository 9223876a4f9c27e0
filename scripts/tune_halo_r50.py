"""Loop tuning with the halo mode on the R50 stride-1 3x3 layers: for each,
time the tune-cache cfg against every halo tile x BLOCK_N x CTA pair (layouts
unchanged) and write the faster cfg back to tune_cache.jsonl.
usage: tune_halo_r50.py N [OUT]"""
import itertools
import json
import os
import shutil
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt  # noqa: E402
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import tunecache  # noqa: E402
from scripts.exptime import timeit  # noqa: E402

N = int(sys.argv[1])
S = bench.LayerSet(N, torch.device("cuda", 0))
cache = tunecache._load()
for l in S.layers:
    L = l["L"]
    if L.R != 3 or L.stride != 1:
        continue
    Ho, Wo = L.out_hw()
    f = lambda c: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"],  # noqa: E731
                             bias=l["bi"], act="relu", cfg=c)
    best = (timeit(lambda: f(l["cfg"])), l["cfg"])
    base = best[0]
    for tw in (16, 32, 64):
        for th in (1, 2, 4, 8):
            if tw < Wo + 2 or 128 % (tw * th) or 128 // (tw * th) > N:
                continue
            for bn, pr in itertools.product((64, 128, 256), (0, 2)):
                if bn > max(64, L.K):
                    continue
                c = {"path": 1, "block_n": bn, "cta_pair": pr, "tile_n": 128 // (tw * th), "tile_h": th,
                     "tile_w": tw, "block_k": 1}
                try:
                    t = timeit(lambda: f(c))
                except alt.AltError:
                    continue
                if alt.last_plan()["block_k"] == 1 and t < best[0]:
                    best = (t, dict(alt.last_plan()))
    print(f"{L.name}: tuned {base:.2f} us -> {best[0]:.2f} us {best[1]}", flush=True)
    if best[1] is not l["cfg"]:
        e = cache[tunecache.key("conv2d", L, N)]
        e["cfg"] = best[1]
        e["us_graph"] = round(best[0], 2)
with open(tunecache._PATH, "w") as fo:
    for v in cache.values():
        fo.write(json.dumps(v) + "\n")
if len(sys.argv) > 2:
    shutil.copy(tunecache._PATH, sys.argv[2])
