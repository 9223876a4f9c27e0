"""Per-CTA timeline of one conv layer (build EXTRA=-DALT_DBG_TILE=t, env ALT_TC_DEBUG=1).
usage: exp_dbg5.py LAYER [block_n] [cta_pair] [split_k]"""
import os, sys, ctypes
os.environ["ALT_TC_DEBUG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import _alt
lib = _alt._lib
lib.alt__debug_tc.argtypes = [ctypes.c_void_p, ctypes.c_int64]
names = {38: "sc: item0 DSMEM sum done", 39: "sc: item0 stored", 36: "sc: partial in smem", 37: "sc: after cluster sync", 33: "pro: barriers init", 34: "pro: tmem alloc (warp 1)", 35: "pro: slab table", 32: "prologue done (before griddep wait)", 4: "epi: partial written", 7: "epi: last decided", 0: "start", 1: "setup done", 3: "mma: tile0 committed", 5: "epi: all done", 6: "end",
         24: "prod: before empty wait", 25: "prod: after empty wait", 26: "mma: before tempty", 27: "mma: after tempty",
         28: "mma: first full", 29: "mma: commit tfull", 2: "epi: tfull", 30: "epi: sb staged", 8: "epi: c0 ld",
         9: "epi: c0 math", 10: "epi: c0 smem", 11: "epi: c0 store", 31: "epi: tile end"}
S = bench.LayerSet(int(os.environ.get("BATCH", "32")), torch.device("cuda", 0))
for name in sys.argv[1].split(","):
    l = [l for l in S.layers if l["L"].name == name][0]
    cfg = dict(l["cfg"])
    if len(sys.argv) > 2: cfg["block_n"] = int(sys.argv[2])
    if len(sys.argv) > 3: cfg["cta_pair"] = int(sys.argv[3])
    if len(sys.argv) > 4: cfg["split_k"] = int(sys.argv[4])
    if len(sys.argv) > 5: cfg["split_cluster"] = int(sys.argv[5])
    f = lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"], bias=l["bi"], act="relu", cfg=cfg)
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    if os.environ.get("ISOLATED"):  # one launch on an idle GPU
        lib.alt__debug_tc.restype = ctypes.c_int
        torch.cuda._sleep(1000000)
        f()
        torch.cuda.synchronize()
    ncta = 148
    print('timeit us', round(__import__('scripts.exptime', fromlist=['timeit']).timeit(f), 2))
    buf = np.zeros(ncta * 40, np.uint64)
    lib.alt__debug_tc(buf.ctypes.data, ncta * 40)
    t = buf.reshape(ncta, 40).astype(np.int64)
    # only the CTAs of the last launch (slots of unused CTAs hold older stamps)
    last = t[:, 0].max()
    t = t[t[:, 0] > last - 200_000]
    t0 = t[:, 0][t[:, 0] > 0].min()
    rel = np.where(t > 0, (t - t0) / 1000.0, np.nan)
    print(name, alt.last_plan())
    for k in sorted(names, key=lambda k: np.nanmedian(rel[:, k]) if np.isfinite(rel[:, k]).any() else 1e9):
        col = rel[:, k]
        if not np.isfinite(col).any(): continue
        print(f"   {names[k]:26s} min {np.nanmin(col):8.2f} med {np.nanmedian(col):8.2f} max {np.nanmax(col):8.2f}")
