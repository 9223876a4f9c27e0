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
            "config": config}
    line.update(extra)
    return line


def run(args):
    ws, rank, local = bench.dist_init()
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    out = None
    if args.workload in ("r18", "mv2"):
        if args.workload == "r18":
            global_batch = 256
            lo, hi = D.shard_range(global_batch, rank, ws)
            ch = CH.resnet18(hi - lo, dev)
        else:
            global_batch = 16 * ws
            ch = CH.mobilenet_v2(16, dev)
        gathered = {}

        def step():
            y = ch.run()
            if args.workload == "r18" and ws > 1:
                gathered["y"] = D.gather_outputs(y, ws)   # the only cross-GPU step

        n0 = alt.launch_count()
        step()
        torch.cuda.synchronize()
        per_step_launches = alt.launch_count() - n0
        ms = _time(step, args.steps, args.warmup, ws, graph=(ws == 1 or args.workload != "r18"))
        flops = ch.flops * (global_batch / ch.N if args.workload == "r18" else ws)
        recorded, launched = ch.plan()
        cfg = {"workload": ("ResNet-18 conv chain (conv1 7x7 + 16 3x3 + 3 1x1 ds, maxpool, BN+ReLU, "
                            "residual adds), global batch 256 sharded by batch, NCCL all-gather of the "
                            "512x7x7 output" if args.workload == "r18" else
                            "MobileNet-V2 chain (52 convs, 17 depthwise, BN+ReLU6, residual adds), "
                            "batch 16 per GPU"),
               "global_batch": global_batch, "per_gpu_batch": ch.N, "parallelism": f"dp{ws}"}
        out = _line(args, ws, flops / (ms * 1e-3) / 1e12, "TFLOP/s", ms, cfg,
                    {"scaling": "strong" if args.workload == "r18" else "weak",
                     "gpu_launches": per_step_launches * args.steps,
                     "propagation": {"alg1_recorded_conversions": recorded,
                                     "standalone_conversion_kernels": launched,
                                     "launches_per_step": per_step_launches,
                                     "ops_per_step": len(ch.ops) + 1}})
    elif args.workload == "bert":
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
            items.append((name, M, N, K, La, a, Lb, b, Lc, c))

        cfgs = {}
        for it in items:
            c = dict(tunecache.lookup_gemm(it[1], it[2], it[3]) or {"path": 1, "block_n": 256})
            c.pop("b_nt", None)  # a layout parameter, not a kernel one
            cfgs[(it[1], it[2], it[3])] = c

        def step():
            for (_, M_, N_, K_, La, a, Lb, b, Lc, c) in items:
                alt.matmul(M_, N_, K_, La, a, Lb, b, Lc, c, cfg=cfgs[(M_, N_, K_)])

        ms = _time(step, args.steps, args.warmup, ws)
        flops = sum(2.0 * M_ * N_ * K_ for (_, M_, N_, K_, *_r) in items) * ws
        per = []
        for it in items:
            t = _time(lambda it=it: alt.matmul(it[1], it[2], it[3], it[4], it[5], it[6], it[7], it[8],
                                               it[9], cfg=cfgs[(it[1], it[2], it[3])]),
                      max(3, args.steps), 2, ws)
            per.append({"gemm": it[0], "M": it[1], "us": round(t * 1e3, 2), "cfg": cfgs[(it[1], it[2], it[3])],
                        "tflops": round(2.0 * it[1] * it[2] * it[3] / (t * 1e-3) / 1e12, 1)})
        out = _line(args, ws, flops / (ms * 1e-3) / 1e12, "TFLOP/s", ms,
                    {"workload": "BERT-base GEMMs at seq 512 x 16 sequences (M=8192): 768x768, "
                                 "768x3072, 3072x768, tiled A M/128 K/64, B N/nt K/64 (nt tuned), C M/128 N/64",
                     "global_batch": 16 * ws, "seq_len": 512, "parallelism": f"dp{ws}"},
                    {"scaling": "weak", "per_gemm": per, "gpu_launches": 3 * args.steps})
    elif args.workload == "relayout":
        from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import relayout_set
        peak = bench.peaks()[1]
        cases, tot_bytes, tot_ms = [], 0.0, 0.0
        for name, shape, sp, dp in relayout_set.cases():
            for dt in (torch.bfloat16, torch.float32):
                S, Dl = alt.Layout(shape, sp), alt.Layout(shape, dp)
                src = S.empty(dt, dev).normal_()
                dst = Dl.empty(dt, dev)
                t = _time(lambda: alt.relayout(S, src, Dl, dst), max(5, args.steps), 2, ws)
                nbytes = relayout_set.alg_bytes(S, Dl, src.element_size())
                gbs = nbytes / (t * 1e-3) / 1e9
                cases.append({"case": name, "dtype": str(dt)[6:], "MB": round(nbytes / 1e6, 1),
                              "us": round(t * 1e3, 1), "GB/s": round(gbs), "frac": round(gbs / peak, 3)})
                tot_bytes += nbytes
                tot_ms += t
        out = _line(args, ws, tot_bytes / (tot_ms * 1e-3) / 1e9, "GB/s", tot_ms, {
            "workload": "D6 relayout set (ResNet tensors at batch 256, BERT A, KCRS weights)",
            "parallelism": f"dp{ws}"}, {"scaling": "weak", "hbm_peak_gbs": peak, "cases": cases})
    if rank == 0 and out is not None:
        print(json.dumps(out))
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()
