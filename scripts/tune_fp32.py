"""Per-layer kernel configuration search for the R50 set in fp32 (the three-
plane path, reading A27): the bf16-tuned configurations were kept for fp32,
but the fp32 reduction is six plane pairs long and the fp32 epilogue has no
cluster / tail split-K forms.  Times, per layer, the bf16 cfg without split,
plain (workspace) split-K 2 / 4 / 8 and BLOCK_N 128 / 256 variants on the
device (CUDA graph replays) and prints the fastest per layer.  Measured
(profiles/r02_fp32_cfg_search.txt): at most 1-3 % per layer and ~1 % on the
set, so bench keeps the bf16 configurations.  Developer tool."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
from bench_layouts import _time_us  # noqa: E402

dev = torch.device("cuda", 0)
S = bench.LayerSet(32, dev, torch.float32)
alt = S.alt
out, log = {}, []
for l in S.layers:
    base = {k: v for k, v in l["cfg"].items() if k not in ("split_k", "split_cluster")}
    cands = [base]
    for sk in (2, 4, 8):
        cands.append(dict(base, split_k=sk, split_cluster=0))
    for bn, pr in ((128, 0), (128, 2), (256, 2)):
        c = dict(base, block_n=bn, cta_pair=pr)
        cands.append(c)
        cands.append(dict(c, split_k=2, split_cluster=0))
    best = None
    for c in cands:
        def fn(c=c):
            alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"], scale=l["sc"], bias=l["bi"],
                       act="relu", cfg=c)
        try:
            fn()
            torch.cuda.synchronize()
            t = _time_us(fn, reps=5, warmup=1)
        except Exception as e:  # noqa: BLE001  (unsupported form for this layer)
            log.append((l["L"].name, c, repr(e)[:80]))
            continue
        log.append((l["L"].name, c, round(t, 1)))
        if best is None or t < best[0]:
            best = (t, c)
    base_t = next((x[2] for x in log if x[0] == l["L"].name and x[1] == base and not isinstance(x[2], str)), None)
    print(f"{l['L'].name:10s} base {base_t} us -> best {best[0]:.1f} us {best[1]}", flush=True)
    out[l["L"].name] = best[1]
