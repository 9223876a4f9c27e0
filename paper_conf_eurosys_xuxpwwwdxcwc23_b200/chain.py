"""Layer chains on ALT layouts with layout propagation (SURVEY §8a rows a5,
a7, a8, a10): ResNet-18 and MobileNet-V2 conv chains (folded BN + ReLU /
ReLU6, residual adds, max-pool) executed through the C-ABI.

Propagation (Alg. 1, plus the producer-side half of Fig. 5b):
every tensor is stored in the input layout its first complex consumer wants;
the producer (a conv's fused epilogue, the pool, or the input "pad" op)
writes that layout directly, so no standalone conversion kernel runs inside
the chain.  `alt_plan_chain` reports where Alg. 1 itself would insert
conversion ops (complex -> complex edges) — here they are fused.
"""
from __future__ import annotations

import json
import math
import os

import torch

from . import _alt as A
from . import layouts as LY
from . import nets, synth


_TUNE_PATH = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "chain_tune.json")


def _numel(shape) -> int:
    n = 1
    for v in shape:
        n *= v
    return n


def chan_tile(C: int) -> int:
    """largest power of two <= 64 dividing C (>= 8 for the tensor-core path)"""
    x = 64
    while x > 1 and C % x:
        x //= 2
    return x


def act_prims(C: int):
    if C % 8:
        Cp = (C + 7) // 8 * 8
        return LY.nchwxc(C, 8, pad_c=Cp - C)
    return LY.nchwxc(C, chan_tile(C))


def block_n(K: int) -> int:
    return 64 if K <= 64 else (128 if K <= 128 else 256)


def wgt_prims(L: nets.ConvShape):
    if L.groups > 1:
        # depthwise: R S K (8 consecutive channels contiguous per tap, read as
        # one 16-byte vector by the depthwise kernel)
        return [("reorder", [1, 2, 3, 0])]
    if L.C % 8:
        return LY.kcrs_wfold(L.K, L.C, L.S)
    x = 8 if L.C % 8 else chan_tile(L.C)
    pad_c = (L.C + 7) // 8 * 8 - L.C if L.C % 8 else 0
    bn = block_n(L.K)
    y = min(L.K, bn)
    while L.K % y:
        y //= 2
    return LY.kcrs_yk_xc(L.K, L.C, y, x, pad_c=pad_c)


class Chain:
    """Device state + launch sequence of one network chain at batch N."""

    def __init__(self, ops, N: int, dev, dtype=torch.bfloat16, name="chain", img_hw=224, policy="propagated"):
        """policy: "propagated" (every tensor in its consumer's tuned layout,
        Alg. 1 + Fig. 5b) or a fixed activation layout for the whole chain,
        "nhwc" / "nchw" (the fixed-layout baseline of P:426-465; weights keep
        their offline layouts)."""
        self.ops, self.N, self.dev, self.dtype = ops, N, dev, dtype
        self.policy = policy
        # logical shapes of every tensor
        shapes = {"img": (N, 3, img_hw, img_hw)}
        for op in ops:
            if op[0] == "conv":
                L = op[1]
                Ho, Wo = L.out_hw()
                shapes[op[5]] = (N, L.K, Ho, Wo)
            else:
                _, k, s, p, src, dst = op
                n, c, h, w = shapes[src]
                shapes[dst] = (n, c, (h + 2 * p - k) // s + 1, (w + 2 * p - k) // s + 1)
        self.shapes = shapes
        # layout of each tensor: the input layout of its first consumer (the
        # same NCHW[x]c family for every consumer here, see act_prims)
        fixed = {"nhwc": LY.nhwc(), "nchw": LY.nchw()}.get(policy)
        if policy != "propagated" and fixed is None:
            raise ValueError(f"unknown layout policy {policy!r}")
        self.layouts = {t: A.Layout(shp, act_prims(shp[1]) if fixed is None else fixed)
                        for t, shp in shapes.items()}
        # a few-channel first conv (C = 3) reads the image window-folded
        # (reading A23): the input pad op writes that layout directly
        L0 = ops[0][1]
        if fixed is None and ops[0][0] == "conv" and ops[0][2] == "img" and L0.C % 8 and L0.groups == 1:
            self.layouts["img"] = A.Layout(shapes["img"], LY.conv_input_wfold(L0.C, L0.S, L0.stride, L0.pad))
        self.img_plain = A.Layout(shapes["img"], [])
        self.buf = {t: torch.zeros(self.layouts[t].phys_shape, dtype=dtype, device=dev) for t in shapes}
        self.img = synth.activations(name + "img", shapes["img"]).to(dtype).to(dev)
        self.launch_ops = []
        gen_w = {}
        for i, op in enumerate(ops):
            if op[0] != "conv":
                continue
            L = op[1]
            wl0 = A.Layout((L.K, L.C // L.groups, L.R, L.S), [])
            wl = A.Layout((L.K, L.C // L.groups, L.R, L.S), wgt_prims(L))
            w0 = synth.weights(name + "w" + L.name, (L.K, L.C // L.groups, L.R, L.S)).to(dtype).to(dev)
            w = torch.zeros(wl.phys_shape, dtype=dtype, device=dev)
            A.relayout(wl0, w0, wl, w)  # weights: converted offline
            sc = synth.bn_scale(name + "s" + L.name, L.K).to(dev)
            bi = synth.bn_bias(name + "b" + L.name, L.K).to(dev)
            gen_w[i] = (wl, w, sc, bi)
        self.weights = gen_w
        # tuned kernel configurations (loop tuning with the layouts fixed by
        # propagation), from chain_tune.json when present
        self.name = name
        self.cfgs = {}
        self.cfgs_loaded = False
        try:
            with open(_TUNE_PATH) as f:
                ent = json.load(f).get(self.tune_key())
            if ent:
                self.cfgs = {int(k): v for k, v in ent.items()}
                self.cfgs_loaded = True
        except (OSError, ValueError):
            pass
        torch.cuda.synchronize(dev) if dev.type == "cuda" else None
        self.flops = sum(op[1].flops(N) for op in ops if op[0] == "conv")

    def min_bytes(self, esize: int = 2) -> float:
        """algorithmic HBM bytes of one pass: every op reads its inputs once
        (a residual too) and writes its output once"""
        tot = 0.0
        for op in self.ops:
            if op[0] == "conv":
                tot += op[1].min_bytes(self.N, esize)
                if op[3] is not None:
                    tot += esize * _numel(self.shapes[op[3]])
            else:
                tot += esize * (_numel(self.shapes[op[4]]) + _numel(self.shapes[op[5]]))
        return tot

    # ------------------------------------------------------------ planning
    def plan(self):
        """Alg. 1 over the chain's DAG via alt_plan_chain.  Returns
        (recorded_conversions, standalone_conversion_launches)."""
        ops = self.ops
        kinds = [0 if op[0] == "conv" else 2 for op in ops] + [2]   # + the input pad op
        pad_op = len(ops)
        producer = {"img": pad_op}
        for i, op in enumerate(ops):
            producer[op[5]] = i
        edges, lays = [], []
        consumed = set()
        for i, op in enumerate(ops):
            srcs = [op[2]] if op[0] == "conv" else [op[4]]
            if op[0] == "conv" and op[3] is not None:
                srcs.append(op[3])  # residual input (slot 1)
            for slot, t in enumerate(srcs):
                n = 1
                for s in self.shapes[t]:
                    n *= s
                p = producer[t]
                edges.append((p, i, slot, n))
                tuned = p < len(ops) and ops[p][0] == "conv"
                lays.append(self.layouts[t] if tuned and not self.layouts[t].identity else None)
                consumed.add(t)
        src_edge, conversion = A.plan_chain(kinds, edges, lays)
        return sum(conversion), 0

    # -------------------------------------------------------------- tuning
    def tune_key(self):
        return f"{self.name}|N{self.N}" + ("" if self.policy == "propagated" else f"|{self.policy}")

    def tune(self, reps=10, warmup=3, store=True, log=None):
        """Per conv op, time candidate kernel configurations (BLOCK_N, CTA
        pair, split-K, output-pixel tile) on the device with every layout
        fixed by propagation (Alg. 1: the downstream layouts are decided, the
        loop schedule is tuned), keep the fastest; stored in chain_tune.json."""
        import itertools
        self.run()
        torch.cuda.synchronize()
        best = {}
        for i, op in enumerate(self.ops):
            if op[0] != "conv" or op[1].groups > 1:
                continue
            L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
            wl, w, sc, bi = self.weights[i]
            p = A.conv_params(self.N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad, L.groups)
            kw = dict(residual=self.buf[res], residual_l=self.layouts[res]) if res is not None else {}
            act = ("relu6" if self._relu6 else "relu") if relu else None
            Ho, Wo = L.out_hw()
            tiles = [None] + [(128 // (th * tw), th, tw) for th in (1, 2, 4) for tw in (4, 8, 16, 32)
                              if tw <= 2 * Wo and th <= 2 * Ho and 128 // (th * tw) <= max(self.N, 1)]
            cands = []
            M = self.N * Ho * Wo
            for bn, pair, sk, t in itertools.product((64, 128, 256), (0, 2), (1, 2, 4, -2, -4), tiles):
                if bn > 64 and bn >= 2 * L.K:
                    continue
                # split-K only where the output tiles leave SMs idle (bounded workspace)
                if abs(sk) > 1 and -(-M // 128) * -(-L.K // bn) > 296:
                    continue
                # cluster split-K (negative): one CTA per tile part, no residual
                if sk < 0 and (pair != 2 or bn < 128 or res is not None):
                    continue
                c = {"path": A.PATH_TC, "block_n": bn, "cta_pair": pair, "split_k": abs(sk),
                     "split_cluster": int(sk < 0)}
                if t is not None:
                    c.update(tile_n=t[0], tile_h=t[1], tile_w=t[2])
                cands.append(c)
            res_t = []
            for c in cands:
                f = lambda c=c: A.conv2d(p, self.layouts[src], self.buf[src], wl, w, self.layouts[dst],
                                         self.buf[dst], scale=sc, bias=bi, act=act, cfg=c, **kw)
                try:
                    for _ in range(warmup):
                        f()
                    torch.cuda.synchronize()
                    # device time without host launch overhead: `reps` launches
                    # captured in a CUDA graph (the plan is cached, so capture
                    # records kernel nodes only)
                    g = torch.cuda.CUDAGraph()
                    cs = torch.cuda.Stream()
                    cs.wait_stream(torch.cuda.current_stream())
                    with torch.cuda.stream(cs), torch.cuda.graph(g, stream=cs):
                        for _ in range(reps):
                            f()
                    torch.cuda.current_stream().wait_stream(cs)
                    g.replay()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    g.replay()
                    e1.record()
                    torch.cuda.synchronize()
                    res_t.append((e0.elapsed_time(e1) / reps * 1e3, c))
                except (A.AltError, RuntimeError):
                    torch.cuda.synchronize()
                    continue
            if res_t:
                res_t.sort(key=lambda t: t[0])
                best[i] = res_t[0][1]
                if log:
                    log(f"op {i} {L.name}: {res_t[0][0]:.1f} us of {len(res_t)} cfgs {res_t[0][1]}")
        self.cfgs = best
        if store:
            try:
                with open(_TUNE_PATH) as f:
                    allc = json.load(f)
            except (OSError, ValueError):
                allc = {}
            allc[self.tune_key()] = {str(k): v for k, v in best.items()}
            with open(_TUNE_PATH, "w") as f:
                json.dump(allc, f, indent=0, sort_keys=True)
        return best

    # ------------------------------------------------------------- running
    def run(self, stream=None):
        """One forward pass: the input pad op converts the image into conv1's
        layout, then every op writes its consumer's layout directly."""
        A.relayout(self.img_plain, self.img, self.layouts["img"], self.buf["img"], stream=stream)
        for i, op in enumerate(self.ops):
            if op[0] == "conv":
                L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
                wl, w, sc, bi = self.weights[i]
                p = A.conv_params(self.N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad, L.groups)
                kw = {}
                if res is not None:
                    kw = dict(residual=self.buf[res], residual_l=self.layouts[res])
                act = ("relu6" if self._relu6 else "relu") if relu else None
                A.conv2d(p, self.layouts[src], self.buf[src], wl, w, self.layouts[dst], self.buf[dst],
                         scale=sc, bias=bi, act=act, stream=stream, cfg=self.cfgs.get(i), **kw)
            else:
                _, k, s, pd, src, dst = op
                n, c, h, w_ = self.shapes[src]
                p = A.conv_params(n, c, h, w_, c, k, k, s, pd)
                A.pool2d(p, self.layouts[src], self.buf[src], self.layouts[dst], self.buf[dst], "max",
                         stream=stream)
        return self.buf[self.ops[-1][5]]

    _relu6 = False

    @property
    def out_name(self):
        return self.ops[-1][5]


def resnet18(N, dev, dtype=torch.bfloat16, img_hw=224, policy="propagated"):
    return Chain(nets.resnet18_chain(img_hw), N, dev, dtype, "r18", img_hw, policy)


def mobilenet_v2(N, dev, dtype=torch.bfloat16, img_hw=224, policy="propagated"):
    c = Chain(nets.mobilenet_v2_chain(img_hw), N, dev, dtype, "mv2", img_hw, policy)
    c._relu6 = True
    return c
