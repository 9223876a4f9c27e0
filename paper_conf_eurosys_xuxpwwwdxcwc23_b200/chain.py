"""Layer chains on ALT layouts with layout propagation (SURVEY §8a rows a5,
a7, a8, a10): ResNet-18 and MobileNet-V2 conv chains (folded BN + ReLU /
ReLU6, residual adds, max-pool) executed through the C-ABI.

Propagation decides the layouts (Alg. 1, with the joint stage of
§6):
  1. every complex op (conv) is tuned on its own by alt_tune at the chain's
     per-GPU batch (`Chain.tune_layouts`, chain_layouts.json "ops"): its
     input x, weight w and output y layouts;
  2. alt_plan_chain runs Alg. 1 with each producer's tuned output layout p_T
     on its out-edges.  Where it inserts a conversion op (complex -> complex
     edge, line 4) this build fuses the conversion into the producer, whose
     epilogue writes the consumer's tuned input layout (Fig. 5b) — but a
     fused conversion moves work into the producer's epilogue (a padded or
     overlapped output layout is written element by element), the B200 form
     of the paper's fusion conflict.  So each converted tensor
     takes the candidate (the consumers' tuned inputs, p_T, the default
     NCHW[x]c) with the lowest MEASURED producer + consumers time
     (`tune_layouts`, chain_layouts.json "tensors"); the first consumer
     (lowest op index) wins ties (the multi-producer rule).
     Tensors Alg. 1 does not convert keep p_T; pools (a conversion boundary,
     reading A10) and the input pad op write their consumer's layout;
  3. the loop schedule of each op is tuned with those layouts fixed
     (`Chain.tune`, chain_tune.json).
No standalone conversion kernel runs inside the chain; `plan()` reports
Alg. 1's recorded conversions and `run()` counts the launches.
"""
from __future__ import annotations

import json
import math
import os

import torch

from . import _alt as A
from . import layouts as LY
from . import nets, synth


_ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
_TUNE_PATH = os.path.join(_ROOT, "chain_tune.json")
_LAYOUT_PATH = os.path.join(_ROOT, "chain_layouts.json")


def _tup(prims):
    """JSON lists -> the binding's primitive tuples"""
    out = []
    for p in prims:
        if p[0] == "split":
            out.append(("split", p[1], list(p[2])))
        elif p[0] == "reorder":
            out.append(("reorder", list(p[1])))
        else:
            out.append(tuple(p))
    return out


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
        self.name = name
        self.tuned, self.tensor_choice = self._load_tuned() if fixed is None else ({}, {})
        self.decisions = {}
        if fixed is None:
            self.layouts = self._propagate()
        else:
            self.layouts = {t: A.Layout(shp, fixed) for t, shp in shapes.items()}
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
            wp = _tup(self.tuned[i]["w"]) if i in self.tuned and self.tuned[i].get("w") else wgt_prims(L)
            wl = A.Layout((L.K, L.C // L.groups, L.R, L.S), wp)
            w0 = synth.weights(name + "w" + L.name, (L.K, L.C // L.groups, L.R, L.S)).to(dtype).to(dev)
            w = torch.zeros(wl.phys_shape, dtype=dtype, device=dev)
            A.relayout(wl0, w0, wl, w)  # weights: converted offline
            sc = synth.bn_scale(name + "s" + L.name, L.K).to(dev)
            bi = synth.bn_bias(name + "b" + L.name, L.K).to(dev)
            gen_w[i] = (wl, w, sc, bi)
        self.weights = gen_w
        # tuned kernel configurations (loop tuning with the layouts fixed by
        # propagation), from chain_tune.json when present
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
    def _graph(self):
        """op kinds (+ the input pad op), edges (producer, consumer, slot,
        numel) and the tensor of each edge"""
        ops = self.ops
        kinds = [0 if op[0] == "conv" else 2 for op in ops] + [2]   # + the input pad op
        pad_op = len(ops)
        producer = {"img": pad_op}
        for i, op in enumerate(ops):
            producer[op[5]] = i
        edges, tens = [], []
        for i, op in enumerate(ops):
            srcs = [op[2]] if op[0] == "conv" else [op[4]]
            if op[0] == "conv" and op[3] is not None:
                srcs.append(op[3])  # residual input (slot 1)
            for slot, t in enumerate(srcs):
                edges.append((producer[t], i, slot, _numel(self.shapes[t])))
                tens.append(t)
        return kinds, edges, tens, producer

    def _default_x(self, i):
        L = self.ops[i][1]
        if self.ops[i][2] == "img" and L.C % 8 and L.groups == 1:
            return LY.conv_input_wfold(L.C, L.S, L.stride, L.pad)   # reading A23
        return act_prims(L.C)

    def _propagate(self):
        """Steps 1-2 of the module docstring: tuned per-op layouts, Alg. 1 via
        alt_plan_chain, conversions fused into the producers."""
        ops = self.ops
        tx, ty = {}, {}
        for i, op in enumerate(ops):
            if op[0] != "conv":
                continue
            L = op[1]
            t = self.tuned.get(i, {})
            tx[i] = _tup(t["x"]) if t.get("x") else self._default_x(i)
            ty[i] = _tup(t["y"]) if t.get("y") else act_prims(L.K)
        kinds, edges, tens, producer = self._graph()
        conv = lambda o: o < len(ops) and ops[o][0] == "conv"  # noqa: E731
        lays = []
        for (p, c, slot, n), t in zip(edges, tens):
            lays.append(A.Layout(self.shapes[t], ty[p]) if conv(p) and ty[p] else None)
        src_edge, conversion = A.plan_chain(kinds, edges, lays)
        self._alg1 = (edges, tens, src_edge, conversion)
        prims = {}
        for t in self.shapes:
            p = producer.get(t)
            cons = [(c, slot, e) for e, ((_, c, slot, _), tt) in enumerate(zip(edges, tens)) if tt == t]
            conv_cons = sorted(c for c, slot, e in cons if slot == 0 and conv(c))
            converted = sorted(c for c, slot, e in cons if slot == 0 and conv(c) and conversion[e])
            if converted and t in self.tensor_choice:
                ch = self.tensor_choice[t]
                prims[t] = _tup(ch["prims"])
                self.decisions[t] = (f"Alg. 1 conversion, measured choice: {ch['choice']}" +
                                     (" (fused into the producer)" if ch["choice"].startswith("consumer") else ""))
            elif converted:
                prims[t] = tx[converted[0]]
                self.decisions[t] = f"Alg. 1 conversion to op {converted[0]}'s tuned input, fused into the producer"
            elif conv(p) if p is not None else False:
                prims[t] = ty[p]
                self.decisions[t] = "producer's tuned output layout p_T"
            elif conv_cons:
                prims[t] = tx[conv_cons[0]]
                self.decisions[t] = ("input pad op" if t == "img" else "pool (conversion boundary)") + \
                    f" writes op {conv_cons[0]}'s tuned input"
            else:
                prims[t] = act_prims(self.shapes[t][1])
                self.decisions[t] = "default"
        self.fused_conversions = sum(1 for t in prims if t in self.decisions and "fused" in self.decisions[t])
        return {t: A.Layout(self.shapes[t], prims[t]) for t in self.shapes}

    def _load_tuned(self):
        try:
            with open(_LAYOUT_PATH) as f:
                ent = json.load(f).get(f"{self.name}|N{self.N}")
        except (OSError, ValueError):
            ent = None
        if not ent or "ops" not in ent:  # untuned, or measured slower than the defaults ("rejected")
            return {}, {}
        return {int(k): v for k, v in ent.get("ops", {}).items()}, ent.get("tensors", {})

    def plan(self):
        """Alg. 1 over the chain's DAG via alt_plan_chain.  Returns
        (recorded_conversions, standalone_conversion_launches): the second is
        measured, launches of one run() minus one per op."""
        kinds, edges, tens, producer = self._graph()
        lays = []
        for (p, c, slot, n), t in zip(edges, tens):
            tuned = p < len(self.ops) and self.ops[p][0] == "conv"
            lays.append(self.layouts[t] if tuned and not self.layouts[t].identity else None)
        src_edge, conversion = A.plan_chain(kinds, edges, lays)
        n0 = A.launch_count()
        self.run()
        launched = A.launch_count() - n0
        expected = 1 + sum(op[1].groups if op[0] == "conv" and 1 < op[1].groups < op[1].C else 1 for op in self.ops)
        return sum(conversion), launched - expected

    def layout_report(self):
        return {t: {"layout": list(self.layouts[t].prims), "why": self.decisions.get(t, self.policy)}
                for t in self.shapes}

    # -------------------------------------------------------------- tuning
    def tune_key(self):
        key = f"{self.name}|N{self.N}" + ("" if self.policy == "propagated" else f"|{self.policy}")
        if self.tuned:  # loop configs belong to the layouts they were tuned on
            import hashlib
            sig = json.dumps({t: [list(map(str, p)) for p in self.layouts[t].prims] for t in sorted(self.shapes)})
            key += "|L" + hashlib.sha1(sig.encode()).hexdigest()[:10]
        return key

    def tune_layouts(self, max_points=24, reps=5, store=True, log=None):
        """Step 1: every conv tuned on its own by alt_tune at this batch (the
        bounded template grid); depthwise convs (no alt_tune
        template) time their NCHW[x]c input tiles directly.  Stored in
        chain_layouts.json; a new Chain then propagates them (step 2)."""
        import itertools
        res = {}
        for i, op in enumerate(self.ops):
            if op[0] != "conv":
                continue
            L = op[1]
            p = A.conv_params(self.N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad, L.groups)
            Ho, Wo = L.out_hw()
            if L.groups == 1 and L.C % 8 == 0:
                its = [t for t in (64, 32, 16) if L.C % t == 0][:2]
                ots = [t for t in (64, 32) if L.K % t == 0]
                bns = [64] if L.K <= 64 else ([128, 256] if L.K >= 256 else [128])
                sp = {0: its, 1: ots, 6: bns, 7: [0, 1] if L.pad else [0]}
                if L.R > 1 and Ho >= 14:
                    sp[8] = [0, 7 if Ho % 7 == 0 else 8]
                    sp[9] = [0, 7 if Wo % 7 == 0 else 8]
                try:
                    r = A.tune("conv2d", p, A.ALT_BF16, sp, max_points=max_points, warmup=2, reps=reps)
                except A.AltError:
                    continue
                res[i] = {"x": r["x"], "w": r["w"], "y": r["y"], "us": r["best_us"], "cfg": r["cfg"]}
                if log:
                    log(f"op {i} {L.name}: {r['best_us']:.1f} us, {r['measured']} points, x {r['x']}")
            elif L.groups == L.C == L.K:
                best = None
                for x in (t for t in (8, 16, 32, 64) if L.C % t == 0):
                    xl = A.Layout((self.N, L.C, L.H, L.W), LY.nchwxc(L.C, x))
                    yl = A.Layout((self.N, L.K, Ho, Wo), LY.nchwxc(L.K, x))
                    xb, yb = xl.empty(self.dtype, self.dev), yl.empty(self.dtype, self.dev)
                    wl, w, sc, bi = self.weights[i]
                    f = lambda: A.conv2d(p, xl, xb, wl, w, yl, yb, scale=sc, bias=bi, act="relu6")  # noqa: E731
                    us = _graph_time(f, 10, 2)
                    if best is None or us < best[0]:
                        best = (us, LY.nchwxc(L.C, x), LY.nchwxc(L.K, x))
                if best:
                    res[i] = {"x": best[1], "y": best[2], "us": best[0]}
                    if log:
                        log(f"op {i} {L.name} (depthwise): {best[0]:.1f} us, x {best[1]}")
        tens = self._choose_tensor_layouts(res, log)
        if store:
            try:
                with open(_LAYOUT_PATH) as f:
                    allc = json.load(f)
            except (OSError, ValueError):
                allc = {}
            allc[f"{self.name}|N{self.N}"] = {"ops": {str(k): v for k, v in res.items()}, "tensors": tens}
            with open(_LAYOUT_PATH, "w") as f:
                json.dump(allc, f, indent=0, sort_keys=True)
        return res

    def _choose_tensor_layouts(self, tuned, log=None):
        """Step 2's measured choice for every tensor Alg. 1 converts: time the
        producer writing each candidate layout plus every conv consumer
        reading it (with the ops' tuned weights / other layouts), keep the
        cheapest."""
        ops = self.ops
        kinds, edges, tens, producer = self._graph()
        conv = lambda o: o < len(ops) and ops[o][0] == "conv"  # noqa: E731
        act = lambda op: ("relu6" if self._relu6 else "relu") if op[4] else None  # noqa: E731
        wts = {}
        for i, op in enumerate(ops):
            if conv(i):
                L = op[1]
                t = tuned.get(i, {})
                wp = _tup(t["w"]) if t.get("w") else wgt_prims(L)
                wl0 = A.Layout((L.K, L.C // L.groups, L.R, L.S), [])
                wl = A.Layout((L.K, L.C // L.groups, L.R, L.S), wp)
                wb = wl.empty(self.dtype, self.dev)
                A.relayout(wl0, torch.zeros(wl0.phys_shape, dtype=self.dtype, device=self.dev), wl, wb)
                wts[i] = (wl, wb)
        def own_x(i):
            t = tuned.get(i, {})
            return _tup(t["x"]) if t.get("x") else self._default_x(i)
        def own_y(i):
            t = tuned.get(i, {})
            return _tup(t["y"]) if t.get("y") else act_prims(ops[i][1].K)
        def time_conv(i, xp, yp):
            op = ops[i]
            L = op[1]
            Ho, Wo = L.out_hw()
            xl = A.Layout(self.shapes[op[2]], xp)
            yl = A.Layout(self.shapes[op[5]], yp)
            xb, yb = torch.zeros(xl.phys_shape, dtype=self.dtype, device=self.dev), yl.empty(self.dtype, self.dev)
            p = A.conv_params(self.N, L.C, L.H, L.W, L.K, L.R, L.S, L.stride, L.pad, L.groups)
            wl, wb = wts[i]
            best = float("inf")
            cfg = tuned.get(i, {}).get("cfg")
            for c in ([dict(cfg, path=A.PATH_TC)] if cfg else []) + [None]:
                try:
                    best = min(best, _graph_time(lambda: A.conv2d(p, xl, xb, wl, wb, yl, yb, act=act(op), cfg=c,
                                                                  pads_zero=True), 5, 2))
                except (A.AltError, RuntimeError):
                    torch.cuda.synchronize()
            return best
        out = {}
        for t in self.shapes:
            p = producer.get(t)
            if not conv(p):
                continue
            cons = sorted(c for (pp, c, slot, n), tt in zip(edges, tens) if tt == t and slot == 0 and conv(c))
            if not cons:
                continue
            cands = []
            for label, pr in [(f"consumer op {c}'s tuned input", own_x(c)) for c in cons] + \
                             [("producer's p_T", own_y(p)), ("default NCHW[x]c", act_prims(self.shapes[t][1]))]:
                if all(pr != q for _, q in cands):
                    cands.append((label, pr))
            costs = []
            for label, pr in cands:
                cost = time_conv(p, own_x(p), pr) + sum(time_conv(c, pr, own_y(c)) for c in cons)
                costs.append((cost, label, pr))
            cost, label, pr = min(costs, key=lambda v: v[0])
            out[t] = {"prims": pr, "choice": label, "cost_us": {lb: round(cs, 2) for cs, lb, _ in costs}}
            if log:
                log(f"tensor {t}: {label} ({cost:.1f} us of {[round(c[0], 1) for c in costs]})")
        return out

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
            # halo tiles (stride-1 3x3: a W run of 16 / 32 / 64 >= Wo + 2)
            halo_tiles = [] if (L.R != 3 or L.stride != 1) else \
                [(128 // (th * tw), th, tw) for tw in (16, 32, 64) for th in (1, 2, 4, 8)
                 if tw >= Wo + 2 and 128 % (th * tw) == 0 and 1 <= 128 // (th * tw) <= max(self.N, 1)]
            cands = []
            M = self.N * Ho * Wo
            for bn, pair, t in itertools.product((64, 128, 256), (0, 2), halo_tiles):
                if bn > 64 and bn >= 2 * L.K:
                    continue
                cands.append({"path": A.PATH_TC, "block_n": bn, "cta_pair": pair, "split_k": 1, "split_cluster": 0,
                              "tile_n": t[0], "tile_h": t[1], "tile_w": t[2], "block_k": 1})
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
                                         self.buf[dst], scale=sc, bias=bi, act=act, cfg=c, pads_zero=True, **kw)
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
                # buffers are zero-initialised and written only by their
                # producer through one layout: their pads stay 0
                A.conv2d(p, self.layouts[src], self.buf[src], wl, w, self.layouts[dst], self.buf[dst],
                         scale=sc, bias=bi, act=act, stream=stream, cfg=self.cfgs.get(i), pads_zero=True, **kw)
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


def _graph_time(f, reps=10, warmup=2):
    """device us per call of f: `reps` calls captured in a CUDA graph"""
    for _ in range(warmup):
        f()
    torch.cuda.synchronize()
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
    return e0.elapsed_time(e1) / reps * 1e3


def resnet18(N, dev, dtype=torch.bfloat16, img_hw=224, policy="propagated"):
    return Chain(nets.resnet18_chain(img_hw), N, dev, dtype, "r18", img_hw, policy)


def mobilenet_v2(N, dev, dtype=torch.bfloat16, img_hw=224, policy="propagated"):
    c = Chain(nets.mobilenet_v2_chain(img_hw), N, dev, dtype, "mv2", img_hw, policy)
    c._relu6 = True
    return c
