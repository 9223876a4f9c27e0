"""Fixed-layout baselines: what ALT's layout tuning buys on B200.

The paper's central measurement (§2 Fig. 1; Table 3)
compares the best loop schedule under a FIXED layout with the jointly tuned
layout + schedule.  Here, per operator of BASELINE configs 2-4:

  r50   every ResNet-50 conv at batch 32: the tuned layout (tune cache) vs
        the fixed NHWC / KRSC / NHWC and NCHW / KCRS / NCHW layouts, each
        with its kernel configuration tuned over the same loop grid
  bert  the BERT-base GEMMs at M = 8192: the tuned tiled layouts vs the
        fixed row-major A with B row-major (KN), B column-major (NK) and the
        NKn layouts of reading A12
  chain the MobileNet-V2 chain (batch 16) with propagated NCHW[x]c layouts
        vs the same chain with every activation fixed to NHWC or NCHW

Every point runs through the public C-ABI (alt_conv2d / alt_matmul) on
whatever path the library picks for that layout (`path` in the result: 1 =
tensor cores, 2 = CUDA-core generic); a layout the tensor-core path cannot
read is a real cost of that layout, not a measurement artefact.
"""
from __future__ import annotations

import itertools

import torch

from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets, synth


def _time_us(fn, reps=10, warmup=2):
    """device us per call: `reps` calls captured in a CUDA graph, replayed."""
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s), torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    g.replay()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


def _best(fn_for_cfg, cfgs, reps):
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    best = None
    for c in cfgs:
        try:
            t = _time_us(lambda: fn_for_cfg(c), reps)
            plan = alt.last_plan()
        except (alt.AltError, RuntimeError):
            torch.cuda.synchronize()
            continue
        if best is None or t < best[0]:
            best = (t, c, plan)
    return best


# loop grid shared by every fixed layout: BLOCK_N x CTA pair (the output-pixel
# tile is the planner's choice); path 0 = whatever path the layout admits
LOOP_GRID = [{"path": 0, "block_n": bn, "cta_pair": pr} for bn, pr in itertools.product((64, 128, 256), (0, 2))
             if not (bn == 64 and pr == 0)]

FIXED_CONV = {
    "NHWC": (LY.nhwc(), [("reorder", [0, 2, 3, 1])], LY.nhwc()),
    "NCHW": ([], [], []),
}


def r50(dev, steps=10, N=32):
    import bench
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    S = bench.LayerSet(N, dev)
    rows = []
    tot = {"tuned": 0.0}
    for l in S.layers:
        L = l["L"]
        Ho, Wo = L.out_hw()
        kw = dict(scale=l["sc"], bias=l["bi"], act="relu")
        t_tuned = _time_us(lambda: alt.conv2d(l["p"], l["lx"], l["x"], l["lw"], l["w"], l["ly"], l["y"],
                                              cfg=l["cfg"], **kw), steps)
        row = {"layer": L.name, "tuned_us": round(t_tuned, 2), "tuned_path": alt.last_plan()["path"]}
        tot["tuned"] += t_tuned
        x0 = l["x0d"]
        w0 = synth.weights("r50w" + L.name, (L.K, L.C, L.R, L.S)).to(torch.bfloat16).to(dev)
        for name, (xp, wp, yp) in FIXED_CONV.items():
            lx = alt.Layout((N, L.C, L.H, L.W), xp)
            lw = alt.Layout((L.K, L.C, L.R, L.S), wp)
            ly = alt.Layout((N, L.K, Ho, Wo), yp)
            x, w, y = lx.empty(torch.bfloat16, dev), lw.empty(torch.bfloat16, dev), ly.empty(torch.bfloat16, dev)
            alt.relayout(l["lx0"], x0, lx, x)
            alt.relayout(alt.Layout((L.K, L.C, L.R, L.S), []), w0, lw, w)
            cfgs = [c for c in LOOP_GRID if c["block_n"] <= max(64, L.K)]
            b = _best(lambda c: alt.conv2d(l["p"], lx, x, lw, w, ly, y, cfg=c, **kw), cfgs, steps)
            if b is None:
                row[name] = None
                continue
            row[name] = {"us": round(b[0], 2), "path": b[2]["path"], "block_n": b[2]["block_n"],
                         "speedup_of_tuned": round(b[0] / t_tuned, 3)}
            tot[name] = tot.get(name, 0.0) + b[0]
            del x, y, w
        rows.append(row)
    flops = S.flops
    summary = {k: {"us": round(v, 1), "tflops": round(flops / (v * 1e-6) / 1e12, 1)} for k, v in tot.items()}
    for k in summary:
        if k != "tuned":
            summary[k]["tuned_speedup"] = round(tot[k] / tot["tuned"], 3)
    del S
    torch.cuda.empty_cache()
    return {"config": f"ResNet-50 conv set, batch {N}, BN+ReLU epilogue", "summary": summary, "layers": rows}


def bert(dev, steps=10, M=8192):
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import tunecache
    rows = []
    tot = {}
    for name, K, N in nets.BERT_GEMMS:
        tuned = dict(tunecache.lookup_gemm(M, N, K) or {"path": 1, "block_n": 256})
        nt = tuned.pop("b_nt", 256)
        A0 = torch.randn(M, K, device=dev).to(torch.bfloat16)
        B0 = torch.randn(K, N, device=dev).to(torch.bfloat16)
        variants = {
            "tuned (A M/128 K/64, B N/nt K/64, C M/128 N/64)":
                (LY.gemm_a_tiled(M, K, 128, 64), LY.gemm_b_tiled_nk(K, N, nt, 64), LY.gemm_c_tiled(M, N, 128, 64),
                 [tuned]),
            "row-major A, B KN (row), C": ([], [], [], LOOP_GRID),
            "row-major A, B NK (col), C": ([], LY.transpose2(), [], LOOP_GRID),
            "NKn (A12: A M/16 K 16, B N/16 K 16, C M/16 N/16 16 16)":
                ([("split", 0, [M // 16, 16]), ("reorder", [0, 2, 1])], LY.gemm_nkn_b(K, N, 16),
                 LY.gemm_c_tiled(M, N, 16, 16), LOOP_GRID),
        }
        row = {"gemm": name}
        for vname, (ap, bp, cp, cfgs) in variants.items():
            La, Lb, Lc = alt.Layout((M, K), ap), alt.Layout((K, N), bp), alt.Layout((M, N), cp)
            a, b, c = La.empty(torch.bfloat16, dev), Lb.empty(torch.bfloat16, dev), Lc.empty(torch.bfloat16, dev)
            alt.relayout(alt.Layout((M, K), []), A0, La, a)
            alt.relayout(alt.Layout((K, N), []), B0, Lb, b)
            bst = _best(lambda cf: alt.matmul(M, N, K, La, a, Lb, b, Lc, c, cfg=cf), cfgs, steps)
            if bst is None:
                row[vname] = None
                continue
            row[vname] = {"us": round(bst[0], 2), "path": bst[2]["path"],
                          "tflops": round(2.0 * M * N * K / (bst[0] * 1e-6) / 1e12, 1)}
            tot[vname] = tot.get(vname, 0.0) + bst[0]
        rows.append(row)
    flops = sum(2.0 * M * N * K for _, K, N in nets.BERT_GEMMS)
    return {"config": f"BERT-base GEMMs, M = {M}",
            "summary": {k: {"us": round(v, 1), "tflops": round(flops / (v * 1e-6) / 1e12, 1)} for k, v in tot.items()},
            "gemms": rows}


def chain(dev, steps=10, N=16):
    """propagated chain layouts vs every activation fixed to one layout"""
    from bench_workloads import _time
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
    out = {}
    for policy in ("propagated", "nhwc", "nchw"):
        try:
            ch = CH.mobilenet_v2(N, dev, policy=policy)
            ms = _time(ch.run, steps, 2, 1)
            out[policy] = {"ms": round(ms, 4), "tflops": round(ch.flops / (ms * 1e-3) / 1e12, 2)}
            del ch
        except Exception as e:  # a layout no kernel reads is a result, not a crash
            out[policy] = {"error": str(e)[:160]}
        torch.cuda.empty_cache()
    return {"config": f"MobileNet-V2 chain, batch {N}", "policies": out}


def run_all(dev, steps=10):
    res = {"r50_b32": r50(dev, steps), "bert_m8192": bert(dev, steps)}
    res["mv2_b16"] = chain(dev, steps)
    return res


if __name__ == "__main__":
    import json
    import sys
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    fn = {"r50": r50, "bert": bert, "chain": chain, "all": run_all}[which]
    print(json.dumps(fn(dev)))
