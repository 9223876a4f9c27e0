"""Steps 1 + 3 of chain.py's propagation for the bench chains: per-op layout
tuning (alt_tune at the per-GPU batch) -> chain_layouts.json, then loop
tuning with the propagated layouts fixed -> chain_tune.json.  Prints the
chain time with the heuristic layouts (before) and the propagated tuned
layouts (after).  usage: tune_chain_layouts.py OUTDIR [name:N ...]"""
import json
import os
import shutil
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH  # noqa: E402

dev = torch.device("cuda", 0)
out = sys.argv[1]
jobs = [a.split(":") for a in sys.argv[2:]] or [["r18", "256"], ["mv2", "16"], ["r18", "32"], ["r18", "64"],
                                                 ["r18", "128"], ["mv2", "1"]]
mk = lambda name, N: CH.resnet18(N, dev) if name == "r18" else CH.mobilenet_v2(N, dev)  # noqa: E731
summary = {}
for name, N in jobs:
    N = int(N)
    t0 = time.time()
    ch = mk(name, N)
    before = CH._graph_time(ch.run, 10, 3)
    ch.tune_layouts(log=lambda m: print(name, N, m, flush=True))
    del ch
    torch.cuda.empty_cache()
    ch = mk(name, N)
    print(name, N, "decisions:", json.dumps({t: d["why"] for t, d in ch.layout_report().items()})[:2000], flush=True)
    mid = CH._graph_time(ch.run, 10, 3)
    ch.tune(log=lambda m: print(name, N, m, flush=True))
    after = CH._graph_time(ch.run, 10, 3)
    kept = after <= before * 1.02
    summary[f"{name}|N{N}"] = {"heuristic_us": round(before, 1), "propagated_untuned_loops_us": round(mid, 1),
                               "propagated_tuned_us": round(after, 1), "fused_conversions": ch.fused_conversions,
                               "kept": kept, "seconds": round(time.time() - t0)}
    if not kept:  # measured slower end to end: the chain keeps the heuristic layouts
        with open(CH._LAYOUT_PATH) as f:
            allc = json.load(f)
        allc[f"{name}|N{N}"] = {"rejected": summary[f"{name}|N{N}"]}
        with open(CH._LAYOUT_PATH, "w") as f:
            json.dump(allc, f, indent=0, sort_keys=True)
    print(name, N, summary[f"{name}|N{N}"], flush=True)
    del ch
    torch.cuda.empty_cache()
    shutil.copy(CH._LAYOUT_PATH, out)
    shutil.copy(CH._TUNE_PATH, out)
    with open(os.path.join(out, "chain_tuning_summary.json"), "w") as f:
        json.dump(summary, f, indent=1)
