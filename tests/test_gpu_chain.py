"""GPU chains with layout propagation: ResNet-18
and MobileNet-V2 conv chains on small images, checked layer by layer against
the fp64 oracle (teacher-forced: each layer's oracle is fed the GPU's own
input of that layer), zero standalone conversion launches
inside the chain, pooling parity, and alt_tune on a small conv."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import chain as CH
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth
from tests.helpers import BF16_TOL, make_operand, norm_rel, read_output, words

pytestmark = pytest.mark.gpu


def _check_chain(ch: CH.Chain, relu6: bool, min_recorded: int = 1):
    dev = torch.device("cuda")
    n0 = alt.launch_count()
    ch.run()
    torch.cuda.synchronize()
    launches = alt.launch_count() - n0
    # one launch per op plus the input "pad" op that converts the image
    # (Fig. 5b): no standalone conversion kernel inside the chain
    assert launches == len(ch.ops) + 1, launches
    recorded, launched = ch.plan()
    assert recorded >= min_recorded and launched == 0, (recorded, launched)
    worst = 0.0
    for i, op in enumerate(ch.ops):
        if op[0] == "conv":
            L, src, res, relu, dst = op[1], op[2], op[3], op[4], op[5]
            wl, w, sc, bi = ch.weights[i]
            Ox = oracle.Layout(ch.shapes[src], ch.layouts[src].prims)
            Ow = oracle.Layout(wl.logical_shape, wl.prims)
            pd = dict(N=ch.N, C=L.C, H=L.H, W=L.W, K=L.K, R=L.R, S=L.S, stride_h=L.stride,
                      stride_w=L.stride, pad_h=L.pad, pad_w=L.pad, groups=L.groups)
            kw = {}
            if res is not None:
                kw = dict(res_l=oracle.Layout(ch.shapes[res], ch.layouts[res].prims),
                          residual=words(ch.buf[res]).reshape(ch.layouts[res].phys_shape))
            act = (2 if relu6 else 1) if relu else 0
            ref = oracle.conv2d(pd, Ox, words(ch.buf[src]).reshape(Ox.phys_shape), Ow,
                                words(w).reshape(Ow.phys_shape), scale=sc.double().cpu().numpy(),
                                bias=bi.double().cpu().numpy(), act=act, **kw)
            got = read_output(oracle.Layout(ch.shapes[dst], ch.layouts[dst].prims), ch.buf[dst],
                              torch.bfloat16)
            err = norm_rel(got, ref)
            worst = max(worst, err)
            assert err <= BF16_TOL, (L.name, err)
        else:
            _, k, s, p, src, dst = op
            Ox = oracle.Layout(ch.shapes[src], ch.layouts[src].prims)
            xin = Ox.read_f64(words(ch.buf[src]))
            ref = oracle.pool2d_f64(xin, k, k, s, p, "max")
            got = read_output(oracle.Layout(ch.shapes[dst], ch.layouts[dst].prims), ch.buf[dst],
                              torch.bfloat16)
            assert np.array_equal(got, ref)   # max of bf16 values is exact
    return worst


def test_resnet18_chain_small():
    ch = CH.resnet18(2, torch.device("cuda"), img_hw=64)
    _check_chain(ch, relu6=False)


def test_mobilenet_v2_chain_small():
    ch = CH.mobilenet_v2(2, torch.device("cuda"), img_hw=64)
    _check_chain(ch, relu6=True)


@pytest.mark.parametrize("kind", ["max", "avg"])
def test_pool_parity(kind):
    x = synth.activations("pool" + kind, (2, 32, 17, 15))
    xp = LY.nchwxc(32, 8)
    Ox, xph, xd = make_operand("pool", xp, x, torch.bfloat16)
    Lx = alt.Layout(x.shape, xp)
    yp = LY.nchwxc(32, 16, pad_hw=1)
    Ly = alt.Layout((2, 32, 9, 8), yp)
    y = torch.full(Ly.phys_shape, 7.0, dtype=torch.bfloat16, device="cuda")
    alt.pool2d(alt.conv_params(2, 32, 17, 15, 32, 3, 3, 2, 1), Lx, xd, Ly, y, kind)
    torch.cuda.synchronize()
    ref = oracle.pool2d_f64(Ox.read_f64(xph), 3, 3, 2, 1, kind)
    got = read_output(oracle.Layout((2, 32, 9, 8), yp), y, torch.bfloat16)
    if kind == "max":
        assert np.array_equal(got, ref)
    else:  # fp32 mean rounded once to bf16
        assert norm_rel(got, ref) <= 4e-3


def _check_tuned_conv(p, N, C, H, K, R, pad, res, stride=1):
    """the tuner's winner: a valid layout pair whose conv is oracle-exact"""
    x = synth.activations("tunex", (N, C, H, H))
    w = synth.weights("tunew", (K, C, R, R))
    Ho = (H + 2 * pad - R) // stride + 1
    Ox, xph, xd = make_operand("tunex", res["x"], x, torch.bfloat16)
    Ow, wph, wd = make_operand("tunew", res["w"], w, torch.bfloat16)
    Ly = alt.Layout((N, K, Ho, Ho), res["y"])
    y = torch.zeros(Ly.phys_shape, dtype=torch.bfloat16, device="cuda")
    alt.conv2d(p, alt.Layout(x.shape, res["x"]), xd, alt.Layout(w.shape, res["w"]), wd, Ly, y, cfg=res["cfg"])
    torch.cuda.synchronize()
    ref = oracle.conv2d(dict(N=N, C=C, H=H, W=H, K=K, R=R, S=R, pad_h=pad, pad_w=pad, stride_h=stride,
                             stride_w=stride), Ox, xph, Ow, wph)
    got = read_output(oracle.Layout((N, K, Ho, Ho), res["y"]), y, torch.bfloat16)
    assert norm_rel(got, ref) <= BF16_TOL


@pytest.mark.parametrize("space", [
    {8: [7], 9: [7]},                         # overlapped input tiles + tiled output (ht = wt = 7)
    {8: [14], 9: [2]},
    {11: [1]},                                # the paper's weight order it' ot' (MN-major B)
    {10: [3], 3: [1]},                        # 3-stage ring, BLOCK_M 256
    {8: [7, 0], 9: [7, 0], 11: [0, 1], 10: [0, 4], 3: [0, 2]},   # mixed grid
], ids=["ht7wt7", "ht14wt2", "paper-w", "stages3-bm256", "mixed"])
def test_tune_conv_template_knobs(space):
    """the widened grid: spatial layout tiles, the
    paper's weight order, BLOCK_M and ring stages; every returned winner is
    a valid layout pair whose conv is oracle-exact"""
    p = alt.conv_params(4, 64, 14, 14, 128, 3, 3, 1, 1)
    sp = {0: [64], 1: [64], 6: [128]}
    sp.update(space)
    res = alt.tune("conv2d", p, alt.ALT_BF16, sp, max_points=32, warmup=1, reps=3)
    assert res["measured"] >= 1 and res["best_us"] > 0
    if 8 in space and space[8][0]:
        assert any(q[0] == "unfold" for q in res["x"]) or len(space[8]) > 1
    _check_tuned_conv(p, 4, 64, 14, 128, 3, 1, res)


def test_tune_conv_two_level_output_template():
    """the two-level output template N H/(h't ht) W/(w't wt) K/(o't ot)
    h't w't o't ht wt ot is a measured grid point; the winner
    restricted to it is oracle-exact"""
    p = alt.conv_params(2, 64, 28, 28, 64, 3, 3, 1, 1)
    res = alt.tune("conv2d", p, alt.ALT_BF16, {0: [64], 1: [8], 6: [64], 8: [7], 9: [7], 12: [2], 13: [2], 14: [2]},
                   max_points=4, warmup=1, reps=3)
    assert res["measured"] >= 1
    split_y = [q for q in res["y"] if q[0] == "split"]
    assert len(split_y) == 3 and all(len(q[2]) == 3 for q in split_y)
    _check_tuned_conv(p, 2, 64, 28, 64, 3, 1, res)


def test_tune_conv_strided_spatial_template():
    p = alt.conv_params(2, 64, 28, 28, 128, 3, 3, 2, 1)
    res = alt.tune("conv2d", p, alt.ALT_BF16, {0: [64], 1: [64], 6: [128], 8: [7], 9: [7]}, max_points=4,
                   warmup=1, reps=3)
    _check_tuned_conv(p, 2, 64, 28, 128, 3, 1, res, stride=2)


def test_tune_conv_small():
    """alt_tune (bounded grid, parity unpinned A19): the winner is a valid
    layout pair whose conv is oracle-exact; the returned time is the
    re-measured median of a finalist."""
    p = alt.conv_params(4, 64, 14, 14, 128, 3, 3, 1, 1)
    res = alt.tune("conv2d", p, alt.ALT_BF16, {0: [64, 32], 1: [64], 6: [128, 256]}, max_points=8,
                   warmup=1, reps=3)
    assert res["measured"] >= 2 and res["best_us"] > 0
    assert res["best_us"] <= 2.0 * min(res["all_us"])
    x = synth.activations("tunex", (4, 64, 14, 14))
    w = synth.weights("tunew", (128, 64, 3, 3))
    Ox, xph, xd = make_operand("tunex", res["x"], x, torch.bfloat16)
    Ow, wph, wd = make_operand("tunew", res["w"], w, torch.bfloat16)
    Ly = alt.Layout((4, 128, 14, 14), res["y"])
    y = torch.zeros(Ly.phys_shape, dtype=torch.bfloat16, device="cuda")
    alt.conv2d(p, alt.Layout(x.shape, res["x"]), xd, alt.Layout(w.shape, res["w"]), wd, Ly, y,
               cfg=res["cfg"])
    torch.cuda.synchronize()
    ref = oracle.conv2d(dict(N=4, C=64, H=14, W=14, K=128, R=3, S=3, pad_h=1, pad_w=1), Ox, xph, Ow, wph)
    got = read_output(oracle.Layout((4, 128, 14, 14), res["y"]), y, torch.bfloat16)
    assert norm_rel(got, ref) <= BF16_TOL


def test_tune_gemm_small():
    g = alt._alt.MatmulParams(512, 256, 256)
    res = alt.tune("matmul", g, alt.ALT_BF16, {0: [128], 1: [64], 2: [128, 256], 6: [256]}, max_points=4,
                   warmup=1, reps=3)
    assert res["measured"] >= 1 and res["best_us"] > 0


@pytest.mark.parametrize("seed", range(80))
def test_pool_random(seed):
    """random max / average pooling (window 1-5, stride 1-3, padding up to
    half the window, odd images, fp32 / bf16) through random layouts (NCHW,
    NHWC, NCHW[x]c, padded, the next conv's pad + unfold template); max is
    bit-exact, average within its single rounding"""
    import random
    rng = random.Random(19000 + seed)
    C = 8 * rng.randint(1, 6)
    N, H, W = rng.randint(1, 3), rng.randint(3, 20), rng.randint(3, 20)
    k = rng.randint(1, 5)
    s = rng.randint(1, 3)
    p = rng.randint(0, k // 2)
    Ho, Wo = (H + 2 * p - k) // s + 1, (W + 2 * p - k) // s + 1
    if Ho < 1 or Wo < 1:
        pytest.skip("empty output")
    kind = rng.choice(["max", "avg"])
    dtype = torch.float32 if rng.random() < 0.3 else torch.bfloat16
    xc, yc = rng.choice([8, 16] if C % 16 == 0 else [8]), rng.choice([8, 16] if C % 16 == 0 else [8])
    xp = rng.choice([[], LY.nhwc(), LY.nchwxc(C, xc), LY.nchwxc(C, xc, pad_hw=1)])
    yps = [[], LY.nhwc(), LY.nchwxc(C, yc), LY.nchwxc(C, yc, pad_hw=rng.randint(1, 2))]
    ht, wt = rng.choice([t for t in (1, 2, 4) if t <= Ho]), rng.choice([t for t in (1, 2, 4) if t <= Wo])
    yps.append(LY.conv_input_tiled(C, yc, Ho, Wo, 3, 3, ht, wt, 1, 1))
    yp = rng.choice(yps)
    x = synth.activations(f"rpool{seed}", (N, C, H, W))
    Ox, xph, xd = make_operand(f"rpool{seed}", xp, x, dtype)
    Ly = alt.Layout((N, C, Ho, Wo), yp)
    y = torch.full(Ly.phys_shape, 7.0, dtype=dtype, device="cuda")
    alt.pool2d(alt.conv_params(N, C, H, W, C, k, k, s, p), alt.Layout(x.shape, xp), xd, Ly, y, kind)
    torch.cuda.synchronize()
    ref = oracle.pool2d_f64(Ox.read_f64(xph), k, k, s, p, kind)
    got = read_output(oracle.Layout((N, C, Ho, Wo), yp), y, dtype)
    if kind == "max":
        assert np.array_equal(got, ref)
    elif dtype == torch.bfloat16:
        assert norm_rel(got, ref) <= 4e-3
    else:
        assert np.max(np.abs(got - ref)) <= 1e-6 * max(1.0, np.max(np.abs(ref)))


@pytest.mark.parametrize("seed", range(40))
def test_chain_random(seed):
    """random layer chains through the Chain runtime (propagated layouts,
    producer epilogues writing their consumers' layouts, residual adds of
    earlier tensors, max pools, depthwise / strided / 1x1 / 3x3 convs): every
    op checked against the oracle on the chain's own buffers, and no
    standalone conversion kernel launched"""
    import random
    from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import nets
    rng = random.Random(21000 + seed)
    img = rng.choice([16, 24, 32])
    C0 = 8 * rng.randint(2, 6)
    ops = [("conv", nets.ConvShape("c0", 3, img, img, C0, 3, 3, 1, 1), "img", None, True, "t0")]
    shapes = {"t0": (C0, img)}
    for i in range(1, rng.randint(3, 8)):
        src = f"t{i - 1}"
        C, H = shapes[src]
        kind = rng.random()
        if kind < 0.15 and H >= 4:
            Ho = (H + 2 - 3) // 2 + 1
            ops.append(("maxpool", 3, 2, 1, src, f"t{i}"))
            shapes[f"t{i}"] = (C, Ho)
            continue
        if kind < 0.35:   # depthwise 3x3
            L = nets.ConvShape(f"dw{i}", C, H, H, C, 3, 3, rng.choice([1, 2]) if H >= 4 else 1, 1, C)
        else:
            R = rng.choice([1, 3])
            s = rng.choice([1, 1, 2]) if H >= 4 else 1
            L = nets.ConvShape(f"c{i}", C, H, H, 8 * rng.randint(2, 8), R, R, s, R // 2)
        Ho, _ = L.out_hw()
        same = [t for t, (c, h) in shapes.items() if c == L.K and h == Ho]
        res = rng.choice(same) if same and rng.random() < 0.4 else None
        ops.append(("conv", L, src, res, rng.random() < 0.7, f"t{i}"))
        shapes[f"t{i}"] = (L.K, Ho)
    ch = CH.Chain(ops, rng.randint(1, 3), torch.device("cuda"), name=f"rch{seed}", img_hw=img)
    _check_chain(ch, relu6=False, min_recorded=0)


@pytest.mark.parametrize("seed", range(30))
def test_tune_random(seed):
    """alt_tune on random convs over random sub-grids (channel tiles, BLOCK_N,
    spatial template ht / wt, weight order, stages, halo): whatever point
    wins, its layouts and configuration give an oracle-exact conv"""
    import random
    rng = random.Random(23000 + seed)
    C = rng.choice([16, 32, 64, 128])
    K = rng.choice([32, 64, 128, 192])
    N, H = rng.randint(1, 4), rng.choice([7, 12, 14, 20, 28])
    R = rng.choice([1, 3])
    stride = rng.choice([1, 1, 2])
    pad = R // 2
    sp = {0: rng.sample([v for v in (8, 16, 32, 64) if C % v == 0], k=1),
          1: rng.sample([v for v in (8, 16, 32, 64) if K % v == 0], k=1),
          6: rng.sample([v for v in (64, 128, 256) if v <= max(64, K)], k=1)}   # BLOCK_N <= K
    Ho = (H + 2 * pad - R) // stride + 1
    if rng.random() < 0.4:
        t = rng.choice([v for v in (2, 4, 7) if Ho % v == 0] or [0])
        if t:
            sp[8], sp[9] = [t], [t]
    if rng.random() < 0.3:
        sp[11] = [0, 1]
    if rng.random() < 0.3:
        sp[10] = [0, rng.choice([2, 3, 4])]
    if R == 3 and stride == 1 and rng.random() < 0.3:
        sp[7] = [0, 1]
    p = alt.conv_params(N, C, H, H, K, R, R, stride, pad)
    try:
        res = alt.tune("conv2d", p, alt.ALT_BF16, sp, max_points=8, warmup=1, reps=2)
    except alt.AltError as e:   # a sub-grid with no tensor-core point (e.g. a ragged
        if e.code != alt._alt.ALT_E_UNSUPPORTED:  # N tile under an MN-major weight order)
            raise
        pytest.skip(str(e))
    assert res["measured"] >= 1 and res["best_us"] > 0
    _check_tuned_conv(p, N, C, H, K, R, pad, res, stride=stride)
