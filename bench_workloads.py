"""The other BASELINE configurations for bench.py (`--workload`):

  r18       config 5: ResNet-18 conv chain, global batch 256 sharded by batch
            across the ranks (strong scaling), final feature map all-gathered
            over NCCL, time = max over ranks of (chain + gather)
  mv2       config 4: MobileNet-V2 chain (depthwise + pointwise) at batch 16
            with layout propagation; reports Alg. 1's recorded conversions vs
            the standalone conversion kernels launched (0)
  bert      config 3: BERT-base GEMMs at seq 512 (M = 8192 = 16 sequences) on
            tiled layouts
  relayout  the D6 set of layout conversions, HBM GB/s per case
  fig12     the paper's Fig. 12 propagation study: pad ->
            C2D 3x3 -> C2D 1x1 at 512 channels (7x7, 14x14), layouts chosen by
            forward propagation (ALT-FP), backward propagation (ALT-BP) or
            independent tuning with the conversion fused into the 3x3's
            epilogue (ALT) or run standalone

Each prints one JSON line like bench.py's.
"""
from __future__ import annotations

import json
import os
import time

import torch

import bench
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import dist as D


def _events():
    return torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def _time(fn, steps, warmup, ws, graph=True):
    """device time per step (ms), max over ranks; fn launches one step."""
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    g = None
    if graph:
        try:
            g = torch.cuda.CUDAGraph()
            s = torch.cuda.Stream()
            s.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(s), torch.cuda.graph(g, stream=s):
                for _ in range(steps):
                    fn()
            torch.cuda.current_stream().wait_stream(s)
        except Exception:
            g = None
    if g is not None and os.environ.get("ALT_BENCH_PREREPLAY", "1") == "1":
        g.replay()  # untimed (more warm-up steps): graph upload, SM clock ramp
        torch.cuda.synchronize()
    bench.barrier(ws)
    torch.cuda.synchronize()
    e0, e1 = _events()
    e0.record()
    if g is not None:
        g.replay()
    else:
        for _ in range(steps):
            fn()
    e1.record()
    torch.cuda.synchronize()
    bench.barrier(ws)
    return bench.max_over_ranks(e0.elapsed_time(e1) / steps, ws)


def _line(args, ws, metric_value, unit, ms, config, extra):
    line = {"metric": bench.METRIC, "value": round(metric_value, 3), "unit": unit, "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4),
            "higher_is_better": True, "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": dict(config, warmup_note="W eager warm-up steps, then one untimed replay of the K-step graph")}
    line.update(extra)
    return line


def r18_strong(steps, warmup, ws, rank, dev, graph=True):
    """BASELINE config 5: the ResNet-18 chain at GLOBAL batch 256, sharded by
    batch over the ws ranks (strong scaling, row a10).  Each rank runs the
    whole chain on its contiguous shard; the final 512x7x7 feature maps are
    all-gathered over NCCL inside the timed region (the path's only
    collective).  Returns a dict (time = max over ranks of chain + gather)."""
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
    global_batch = 256
    lo, hi = D.shard_range(global_batch, rank, ws)
    ch = CH.resnet18(hi - lo, dev)
    gathered = {}

    def step():
        y = ch.run()
        gathered["y"] = D.gather_outputs(y, ws)   # identity at ws = 1
    n0 = alt.launch_count()
    step()
    torch.cuda.synchronize()
    per_step = alt.launch_count() - n0
    ms = _time(step, steps, warmup, ws, graph=graph)
    flops = ch.flops * (global_batch / ch.N)
    recorded, launched = ch.plan()
    out_bytes = gathered["y"].numel() * gathered["y"].element_size()
    return {"workload": "ResNet-18 conv chain (conv1 7x7 + 16 3x3 + 3 1x1 ds, maxpool, BN+ReLU, residual "
                        "adds), global batch 256 sharded by batch, NCCL all-gather of the 512x7x7 output",
            "global_batch": global_batch, "per_gpu_batch": ch.N, "n_gpus": ws, "ms_per_step": round(ms, 4),
            "tflops": round(flops / (ms * 1e-3) / 1e12, 2), "scaling": "strong",
            "gathered_bytes": out_bytes, "gpu_launches_per_step": per_step,
            "cfgs": "chain_tune.json" if ch.cfgs_loaded else "heuristic",
            "propagation": {"alg1_recorded_conversions": recorded, "standalone_conversion_kernels": launched}}


def mv2_chain(steps, warmup, ws, dev, N=16):
    """BASELINE config 4: MobileNet-V2 (52 convs, 17 depthwise) at batch N
    per GPU with layout propagation (Alg. 1)."""
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
    ch = CH.mobilenet_v2(N, dev)
    n0 = alt.launch_count()
    ch.run()
    torch.cuda.synchronize()
    per_step = alt.launch_count() - n0
    ms = _time(ch.run, steps, warmup, ws)
    recorded, launched = ch.plan()
    return {"workload": f"MobileNet-V2 chain (52 convs, 17 depthwise, BN+ReLU6, residual adds), batch {N}",
            "per_gpu_batch": N, "ms_per_step": round(ms, 4), "tflops": round(ch.flops / (ms * 1e-3) / 1e12, 2),
            "hbm_bytes_min": ch.min_bytes(), "hbm_gbs_min": round(ch.min_bytes() / (ms * 1e-3) / 1e9, 1),
            "gpu_launches_per_step": per_step,
            "propagation": {"alg1_recorded_conversions": recorded, "standalone_conversion_kernels": launched}}


def bert_set(steps, warmup, ws, dev, bias="none"):
    """BASELINE config 3: BERT-base GEMMs at M = 8192 on tiled layouts."""
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import tunecache
    M = 8192
    items = []
    for name, K, N in nets.BERT_GEMMS:
        tuned = tunecache.lookup_gemm(M, N, K) or {}
        La = alt.Layout((M, K), LY.gemm_a_tiled(M, K, 128, 64))
        Lb = alt.Layout((K, N), LY.gemm_b_tiled_nk(K, N, tuned.get("b_nt", 256), 64))
        Lc = alt.Layout((M, N), LY.gemm_c_tiled(M, N, 128, 64))
        a, b, c = La.empty(torch.bfloat16, dev).normal_(), Lb.empty(torch.bfloat16, dev).normal_(), \
            Lc.empty(torch.bfloat16, dev)
        bvec = torch.randn(N, device=dev).to(torch.bfloat16)
        if bias == "attached":   # store_at: the bias rides in the weight
            Lz = alt.Layout((K + 1, N), LY.gemm_z_tiled_nk(K, N, tuned.get("b_nt", 256), 64))
            z = Lz.empty(torch.bfloat16, dev)
            alt.store_at(Lb, b, bvec, 0, Lz, z)
            Lb, b = Lz, z
        cfg = dict(tuned or {"path": 1, "block_n": 256})
        cfg.pop("b_nt", None)  # a layout parameter, not a kernel one
        items.append((name, M, N, K, La, a, Lb, b, Lc, c, bvec.float(), cfg))

    def gemm(it):
        _, M_, N_, K_, La, a, Lb, b, Lc, c, bv, cfg = it
        if bias == "attached":
            alt.matmul_store_at(M_, N_, K_, La, a, Lb, b, Lc, c, cfg=cfg)
        else:
            alt.matmul(M_, N_, K_, La, a, Lb, b, Lc, c, bias=bv if bias == "separate" else None, cfg=cfg)

    def step():
        for it in items:
            gemm(it)
    ms = _time(step, steps, warmup, ws)
    flops = sum(2.0 * it[1] * it[2] * it[3] for it in items)
    per = []
    for it in items:
        t = _time(lambda it=it: gemm(it), max(3, steps), 2, ws)
        per.append({"gemm": it[0], "M": it[1], "N": it[2], "K": it[3], "us": round(t * 1e3, 2), "cfg": it[11],
                    "tflops": round(2.0 * it[1] * it[2] * it[3] / (t * 1e-3) / 1e12, 1)})
    return {"workload": "BERT-base GEMMs at seq 512 x 16 sequences (M=8192): 768x768, 768x3072, 3072x768, "
                        "tiled A M/128 K/64, B N/nt K/64 (nt tuned), C M/128 N/64"
                        + {"none": "", "separate": ", fp32 bias vector in the epilogue",
                           "attached": ", bias attached to the weight columns by store_at "
                                       "(Z N/nt (K+64)/64 nt 64), read in place"}[bias],
            "ms_per_step": round(ms, 4), "tflops": round(flops / (ms * 1e-3) / 1e12, 2), "per_gemm": per}


def relayout_run(steps, ws, dev):
    """The D6 relayout set: algorithmic HBM GB/s per case and in aggregate."""
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import relayout_set
    peak = bench.peaks()[1]
    cases, tot_bytes, tot_ms = [], 0.0, 0.0
    for name, shape, sp, dp in relayout_set.cases():
        for dt in (torch.bfloat16, torch.float32):
            S, Dl = alt.Layout(shape, sp), alt.Layout(shape, dp)
            src = S.empty(dt, dev).normal_()
            dst = Dl.empty(dt, dev)
            t = _time(lambda: alt.relayout(S, src, Dl, dst), max(5, steps), 2, ws)
            nbytes = relayout_set.alg_bytes(S, Dl, src.element_size())
            gbs = nbytes / (t * 1e-3) / 1e9
            cases.append({"case": name, "dtype": str(dt)[6:], "MB": round(nbytes / 1e6, 1),
                          "us": round(t * 1e3, 1), "GB/s": round(gbs), "frac": round(gbs / peak, 3)})
            tot_bytes += nbytes
            tot_ms += t
            del src, dst
    return {"workload": "D6 relayout set (ResNet tensors at batch 256, BERT A, KCRS weights)",
            "gbs": round(tot_bytes / (tot_ms * 1e-3) / 1e9, 1), "hbm_peak_gbs": peak,
            "frac": round(tot_bytes / (tot_ms * 1e-3) / 1e9 / peak, 3), "ms": round(tot_ms, 4), "cases": cases}


def run(args):
    ws, rank, local = bench.dist_init()
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    out = None
    if args.workload == "r18":
        r = r18_strong(args.steps, args.warmup, ws, rank, dev)
        out = _line(args, ws, r["tflops"], "TFLOP/s", r["ms_per_step"],
                    {"workload": r["workload"], "global_batch": 256, "per_gpu_batch": r["per_gpu_batch"],
                     "parallelism": f"dp{ws}",
                     "l2": "inputs larger than L2 (R18 chain at batch 256 touches > 1 GB per step)"},
                    {"scaling": "strong", "gpu_launches": r["gpu_launches_per_step"] * args.steps,
                     "propagation": r["propagation"], "gathered_bytes": r["gathered_bytes"]})
    elif args.workload == "mv2":
        r = mv2_chain(args.steps, args.warmup, ws, dev)
        out = _line(args, ws, r["tflops"] * ws, "TFLOP/s", r["ms_per_step"],
                    {"workload": r["workload"], "global_batch": 16 * ws, "per_gpu_batch": 16,
                     "parallelism": f"dp{ws}", "l2": f"inputs larger than L2 ({r['hbm_bytes_min'] / 1e6:.0f} MB "
                                                      "of algorithmic HBM traffic per step)"},
                    {"scaling": "weak", "gpu_launches": r["gpu_launches_per_step"] * args.steps,
                     "propagation": r["propagation"], "hbm_gbs_min": r["hbm_gbs_min"]})
    elif args.workload == "bert":
        r = bert_set(args.steps, args.warmup, ws, dev, args.bert_bias)
        out = _line(args, ws, r["tflops"] * ws, "TFLOP/s", r["ms_per_step"],
                    {"workload": r["workload"], "global_batch": 16 * ws, "seq_len": 512, "parallelism": f"dp{ws}",
                     "l2": "inputs larger than L2 (the three GEMMs touch ~161 MB of A, B and C per step; per_gemm repeats one GEMM, whose operands fit in L2)"},
                    {"scaling": "weak", "per_gemm": r["per_gemm"], "gpu_launches": 3 * args.steps})
    elif args.workload == "relayout":
        r = relayout_run(args.steps, ws, dev)
        out = _line(args, ws, r["gbs"], "GB/s", r["ms"], {"workload": r["workload"], "parallelism": f"dp{ws}",
                                                      "l2": "no flush; each case moves src + dst >= 200 MB except R6 bf16 (101 MB, partly L2-resident across repetitions) and R7 (9.4 MB of weights, the offline a3 transform, L2-resident)"},
                    {"scaling": "weak", "hbm_peak_gbs": r["hbm_peak_gbs"], "cases": r["cases"]})
    elif args.workload == "fig12":
        out = fig12(args, ws)
    if rank == 0 and out is not None:
        print(json.dumps(out))
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


# ------------------------------------------------------------------ Fig. 12 -
def fig12(args, ws):
    """Fig. 12: subgraph pad -> C2D 3x3 (512 -> 512, s1, p1) ->
    C2D 1x1 (512 -> K1) at 7x7 (K1 = 512) and 14x14 (K1 = 2048).  Every
    (layout, kernel configuration) point is timed on the device (CUDA graph
    of repeated launches); the policies combine them as the paper describes:
      ALT-FP  tune the 3x3 (its x and y layouts), the 1x1 reads the 3x3's y
      ALT-BP  tune the 1x1 (its x layout), the 3x3 must write that layout
      ALT     tune both independently; the 1x1's layout is written by the
              3x3's fused epilogue (this build's conversion) or converted by
              a standalone relayout (the paper's conversion op)"""
    import itertools
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth
    dev = torch.device("cuda", 0)
    C = 512
    tiles = (64, 32, 16)
    cfgs = [{"path": 1, "block_n": bn, "cta_pair": pr, "split_k": sk, "split_cluster": scl}
            for bn, pr, (sk, scl) in itertools.product((128, 256), (0, 2), ((1, 0), (2, 0), (2, 1), (4, 1)))
            if not (scl and pr != 2)]

    def tmin(fn_for_cfg):
        best = None
        for c in cfgs:
            try:
                t = _time(lambda: fn_for_cfg(c), 10, 2, 1) * 1e3
            except Exception:
                torch.cuda.synchronize()
                continue
            if best is None or t < best[0]:
                best = (t, c)
        return best

    subs = []
    for (name, H, K1) in (("Sg#1 7x7", 7, 512), ("Sg#2 14x14", 14, 2048)):
        for N in (1, 32):
            x0 = synth.activations(f"f12x{H}", (N, C, H, H)).to(torch.bfloat16).to(dev)
            Lx0 = alt.Layout((N, C, H, H), [])
            w3 = synth.weights("f12w3", (C, C, 3, 3)).to(torch.bfloat16).to(dev)
            w1 = synth.weights(f"f12w1{K1}", (K1, C, 1, 1)).to(torch.bfloat16).to(dev)
            p3, p1 = alt.conv_params(N, C, H, H, C, 3, 3, 1, 1), alt.conv_params(N, C, H, H, K1, 1, 1, 1, 0)
            L3 = {}
            for it in tiles:  # 3x3 input layouts written by the pad op (padding materialised or not)
                for pad in (0, 1):
                    L = alt.Layout((N, C, H, H), LY.nchwxc(C, it, pad_hw=pad))
                    buf = L.empty(torch.bfloat16, dev)
                    alt.relayout(Lx0, x0, L, buf)
                    L3[(it, pad)] = (L, buf)
            Lmid = {t: alt.Layout((N, C, H, H), LY.nchwxc(C, t)) for t in tiles}
            mid = {t: Lmid[t].empty(torch.bfloat16, dev) for t in tiles}
            Ly1 = alt.Layout((N, K1, H, H), LY.nchwxc(K1, 64))
            y1 = Ly1.empty(torch.bfloat16, dev)
            W3, W1 = {}, {}
            for it in tiles:
                for bn in (128, 256):
                    lw = alt.Layout((C, C, 3, 3), LY.kcrs_yk_xc(C, C, bn, it))
                    wt = lw.empty(torch.bfloat16, dev)
                    alt.relayout(alt.Layout((C, C, 3, 3), []), w3, lw, wt)
                    W3[(it, bn)] = (lw, wt)
                    lw1 = alt.Layout((K1, C, 1, 1), LY.kcrs_yk_xc(K1, C, bn, it))
                    wt1 = lw1.empty(torch.bfloat16, dev)
                    alt.relayout(alt.Layout((K1, C, 1, 1), []), w1, lw1, wt1)
                    W1[(it, bn)] = (lw1, wt1)
            torch.cuda.synchronize()
            # pad op (plain NCHW -> the 3x3's input layout)
            t_pad = {k: _time(lambda k=k: alt.relayout(Lx0, x0, L3[k][0], L3[k][1]), 10, 2, 1) * 1e3 for k in L3}
            # C2D 3x3 for every (x layout, y layout); C2D 1x1 for every x layout
            t3 = {}
            for (it, pad), ot in itertools.product(L3.keys(), tiles):
                Lx, xb = L3[(it, pad)]
                t3[(it, pad, ot)] = tmin(lambda c, Lx=Lx, xb=xb, it=it, ot=ot: alt.conv2d(
                    p3, Lx, xb, W3[(it, c["block_n"])][0], W3[(it, c["block_n"])][1], Lmid[ot], mid[ot], cfg=c))
            t1 = {ot: tmin(lambda c, ot=ot: alt.conv2d(p1, Lmid[ot], mid[ot], W1[(ot, c["block_n"])][0],
                                                        W1[(ot, c["block_n"])][1], Ly1, y1, cfg=c)) for ot in tiles}
            t3 = {k: v for k, v in t3.items() if v is not None}
            t1 = {k: v for k, v in t1.items() if v is not None}
            conv = {(a, b): _time(lambda a=a, b=b: alt.relayout(Lmid[a], mid[a], Lmid[b], mid[b]), 10, 2, 1) * 1e3
                    for a in tiles for b in tiles if a != b}
            k3 = lambda k: t3[k][0] + t_pad[k[:2]]  # noqa: E731
            # ALT-FP: best 3x3 point, the 1x1 reads its y layout
            fp3 = min(t3, key=k3)
            fp = (k3(fp3), t1[fp3[2]][0])
            # ALT-BP: best 1x1 point, the 3x3 must write that layout
            ot1 = min(t1, key=lambda o: t1[o][0])
            bp3 = min((k for k in t3 if k[2] == ot1), key=k3)
            bp = (k3(bp3), t1[ot1][0])
            # ALT: independent; fused conversion = the 3x3 (its own x) writes the 1x1's layout
            alt_f3 = min((k for k in t3 if k[:2] == fp3[:2] and k[2] == ot1), key=k3)
            altf = (k3(alt_f3), t1[ot1][0])
            conv_us = conv.get((fp3[2], ot1), 0.0)
            alts = (k3(fp3), conv_us, t1[ot1][0])
            subs.append({"subgraph": name, "batch": N, "K1": K1,
                         "ALT-FP": {"c2d3x3_us": round(fp[0], 2), "c2d1x1_us": round(fp[1], 2),
                                    "total_us": round(sum(fp), 2), "layouts": {"x3": fp3[:2], "y3=x1": fp3[2]}},
                         "ALT-BP": {"c2d3x3_us": round(bp[0], 2), "c2d1x1_us": round(bp[1], 2),
                                    "total_us": round(sum(bp), 2), "layouts": {"x3": bp3[:2], "y3=x1": ot1}},
                         "ALT (fused conversion)": {"c2d3x3_us": round(altf[0], 2), "c2d1x1_us": round(altf[1], 2),
                                                    "total_us": round(sum(altf), 2),
                                                    "layouts": {"x3": alt_f3[:2], "y3": ot1, "x1": ot1}},
                         "ALT (standalone conversion)": {"c2d3x3_us": round(alts[0], 2),
                                                         "conversion_us": round(alts[1], 2),
                                                         "c2d1x1_us": round(alts[2], 2),
                                                         "total_us": round(sum(alts), 2),
                                                         "layouts": {"x3": fp3[:2], "y3": fp3[2], "x1": ot1}}})
    value = sum(s_["ALT (fused conversion)"]["total_us"] for s_ in subs)
    line = _line(args, ws, value, "us", value * 1e-3,
                 {"workload": "Fig. 12 propagation study: pad -> C2D 3x3 512 -> C2D 1x1 (7x7 -> 512, "
                              "14x14 -> 2048), batch 1 and 32, layouts NCHW[x]c x in {64,32,16} with "
                              "optional materialised padding", "parallelism": "dp1"},
                 {"scaling": "weak", "higher_is_better": False, "subgraphs": subs,
                  "note": "value = sum over subgraphs of the ALT (independent tuning, fused conversion) "
                          "totals; pad op time included in the C2D 3x3 column"})
    return line
