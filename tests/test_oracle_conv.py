"""Pins for oracle O3-O6 (conv2d, layout-native conv, GEMM, epilogue).

  * O3 vs torch.nn.functional.conv2d in float64 on CPU (library routine) and
    vs a pure-Python 7-loop brute force on tiny shapes;
  * special cases: a 1x1 conv equals a GEMM (numpy), a one-hot filter is a
    shifted copy, depthwise == per-channel conv;
  * O4 (Eq. (1) on the Fig. 2 overlapped tiles) is bit-exact equal to O3
    (invariant I3, oracle side), including the Table 3 layout of R18 conv1;
  * reading operands through any layout gives bit-identical results
    (invariant I2, oracle side);
  * O5 vs numpy matmul in fp64; O6 closed forms.
"""
import itertools

import numpy as np
import pytest
import torch

import oracle


def _params(N, C, H, W, K, R, S, V=1, pad=0, groups=1):
    return dict(N=N, C=C, H=H, W=W, K=K, R=R, S=S, stride_h=V, stride_w=V,
                pad_h=pad, pad_w=pad, groups=groups)


def _torch_conv(p, x, w):
    return torch.nn.functional.conv2d(
        torch.from_numpy(x), torch.from_numpy(w), stride=(p["stride_h"], p["stride_w"]),
        padding=(p["pad_h"], p["pad_w"]), groups=p["groups"]).numpy()


CASES = [
    _params(1, 16, 14, 14, 32, 3, 3, 1, 1),          # config 1 (D1)
    _params(2, 3, 17, 15, 8, 7, 7, 2, 3),            # conv1-like, stride 2
    _params(3, 8, 9, 9, 8, 1, 1, 2, 0),              # 1x1 stride-2 downsample
    _params(2, 8, 10, 10, 8, 3, 3, 1, 1, groups=8),  # depthwise
    _params(1, 8, 6, 6, 4, 3, 3, 2, 1, groups=2),    # grouped
    _params(2, 5, 5, 7, 3, 2, 3, 1, 0),
]


@pytest.mark.parametrize("p", CASES)
def test_conv_vs_torch_float64(p):
    rng = np.random.default_rng(1)
    x = rng.uniform(-1, 1, (p["N"], p["C"], p["H"], p["W"]))
    w = rng.uniform(-1, 1, (p["K"], p["C"] // p["groups"], p["R"], p["S"]))
    y = oracle.conv2d_f64(p, x, w)
    ref = _torch_conv(p, x, w)
    assert y.shape == ref.shape
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


def _brute(p, x, w):
    N, C, H, W, K, R, S = (p[k] for k in "NCHWKRS")
    V, pd, g = p["stride_h"], p["pad_h"], p["groups"]
    Ho, Wo = (H + 2 * pd - R) // V + 1, (W + 2 * pd - S) // V + 1
    y = np.zeros((N, K, Ho, Wo))
    for n, k, oh, ow in itertools.product(range(N), range(K), range(Ho), range(Wo)):
        grp = k * g // K
        acc = 0.0
        for c, r, s in itertools.product(range(C // g), range(R), range(S)):
            ih, iw = oh * V - pd + r, ow * V - pd + s
            if 0 <= ih < H and 0 <= iw < W:
                acc += x[n, grp * (C // g) + c, ih, iw] * w[k, c, r, s]
        y[n, k, oh, ow] = acc
    return y


def test_conv_vs_python_brute_force_bit_exact():
    for p in [_params(1, 3, 5, 6, 2, 3, 3, 1, 1), _params(2, 4, 5, 5, 4, 3, 3, 2, 1, groups=2)]:
        rng = np.random.default_rng(2)
        x = rng.uniform(-1, 1, (p["N"], p["C"], p["H"], p["W"]))
        w = rng.uniform(-1, 1, (p["K"], p["C"] // p["groups"], p["R"], p["S"]))
        assert np.array_equal(oracle.conv2d_f64(p, x, w), _brute(p, x, w))


def test_conv_1x1_equals_gemm():
    p = _params(2, 12, 5, 4, 7, 1, 1)
    rng = np.random.default_rng(3)
    x = rng.uniform(-1, 1, (2, 12, 5, 4))
    w = rng.uniform(-1, 1, (7, 12, 1, 1))
    y = oracle.conv2d_f64(p, x, w)
    ref = np.einsum("nchw,kc->nkhw", x, w[:, :, 0, 0])
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=1e-13)


def test_conv_one_hot_filter_is_shift():
    p = _params(1, 1, 6, 6, 1, 3, 3, 1, 1)
    x = np.random.default_rng(4).uniform(-1, 1, (1, 1, 6, 6))
    w = np.zeros((1, 1, 3, 3))
    w[0, 0, 2, 0] = 1.0                    # y[p,q] = x[p+1, q-1]
    y = oracle.conv2d_f64(p, x, w)
    ref = np.zeros_like(x)
    ref[0, 0, :5, 1:] = x[0, 0, 1:, :5]
    assert np.array_equal(y, ref)


@pytest.mark.parametrize("V,R,ht,wt,pad,H", [(1, 3, 7, 7, 1, 14), (1, 3, 4, 2, 1, 9),
                                             (2, 3, 3, 4, 1, 13), (2, 1, 2, 2, 0, 8),
                                             (1, 1, 5, 3, 0, 10), (2, 7, 4, 5, 3, 21)])
def test_layout_native_conv_eq1_bit_exact(V, R, ht, wt, pad, H):
    """O4 == O3 bit-exactly (I3): the input is stored as Fig. 2's overlapped
    tiles, pad(H)+pad(W) then unfold(H, V(ht-1)+R, V ht) (reading A6)."""
    N, C, K = 2, 3, 4
    p = _params(N, C, H, H, K, R, R, V, pad)
    rng = np.random.default_rng(5)
    x = rng.uniform(-1, 1, (N, C, H, H)).astype(np.float32)
    w = rng.uniform(-1, 1, (K, C, R, R)).astype(np.float32)
    B, S = V * (ht - 1) + R, V * ht
    Bw, Sw = V * (wt - 1) + R, V * wt
    Lx = oracle.Layout(x.shape, [("pad", 2, pad, pad), ("pad", 3, pad, pad),
                                 ("unfold", 2, B, S), ("unfold", 4, Bw, Sw)])
    xu = Lx.materialize(x.view(np.uint32)).view(np.float32).astype(np.float64)
    y4 = oracle.conv2d_unfold_native(p, ht, wt, xu, w.astype(np.float64))
    y3 = oracle.conv2d_f64(p, x.astype(np.float64), w.astype(np.float64))
    assert np.array_equal(y4, y3)


def test_layout_native_conv_table3_r18_conv1():
    """W11: R18 conv1 (I=3, 224 padded to 230, O=64, 7x7, stride 2) in the
    searched layout ht=4, wt=16 of Table 3; O = 8 here to keep
    the test fast (channel count does not enter Eq. (1))."""
    p = _params(1, 3, 224, 224, 8, 7, 7, 2, 3)
    rng = np.random.default_rng(6)
    x = rng.uniform(-1, 1, (1, 3, 224, 224)).astype(np.float32)
    w = rng.uniform(-1, 1, (8, 3, 7, 7)).astype(np.float32)
    Lx = oracle.Layout(x.shape, [("pad", 2, 3, 3), ("pad", 3, 3, 3),
                                 ("unfold", 2, 13, 8), ("unfold", 4, 37, 32)])
    assert Lx.phys_shape == (1, 3, 29, 13, 8, 37)
    xu = Lx.materialize(x.view(np.uint32)).view(np.float32).astype(np.float64)
    y4 = oracle.conv2d_unfold_native(p, 4, 16, xu, w.astype(np.float64))
    y3 = oracle.conv2d_f64(p, x.astype(np.float64), w.astype(np.float64))
    assert np.array_equal(y4, y3)


XLAYOUTS = [
    [],
    [("reorder", [0, 2, 3, 1])],
    [("split", 1, [2, 4]), ("reorder", [0, 1, 3, 4, 2])],
    [("pad", 2, 1, 1), ("pad", 3, 1, 1), ("unfold", 2, 5, 3), ("unfold", 4, 5, 3),
     ("split", 1, [2, 4]), ("reorder", [0, 3, 5, 1, 4, 6, 2])],
]
WLAYOUTS = [
    [],
    [("split", 0, [2, 4]), ("split", 2, [2, 4]), ("reorder", [0, 2, 4, 5, 1, 3])],  # KCRS4k4c
    [("reorder", [0, 2, 3, 1])],                                                     # KRSC
]


@pytest.mark.parametrize("xi", range(len(XLAYOUTS)))
@pytest.mark.parametrize("wi", range(len(WLAYOUTS)))
@pytest.mark.parametrize("dt", [np.float32, "bf16"])
def test_conv_through_layouts_is_layout_independent(xi, wi, dt):
    """I2 on the oracle side: reading through any layout is exact."""
    p = _params(2, 8, 7, 7, 8, 3, 3, 1, 1)
    rng = np.random.default_rng(7)
    x = rng.uniform(-1, 1, (2, 8, 7, 7)).astype(np.float32)
    w = rng.uniform(-1, 1, (8, 8, 3, 3)).astype(np.float32)
    if dt == "bf16":
        xw = (x.view(np.uint32) >> 16).astype(np.uint16)
        ww = (w.view(np.uint32) >> 16).astype(np.uint16)
        xr, wr = oracle.bf16_bits_to_f64(xw), oracle.bf16_bits_to_f64(ww)
    else:
        xw, ww = x.view(np.uint32), w.view(np.uint32)
        xr, wr = x.astype(np.float64), w.astype(np.float64)
    Lx, Lw = oracle.Layout(x.shape, XLAYOUTS[xi]), oracle.Layout(w.shape, WLAYOUTS[wi])
    y = oracle.conv2d(p, Lx, Lx.materialize(xw), Lw, Lw.materialize(ww))
    assert np.array_equal(y, oracle.conv2d_f64(p, xr, wr))
    pts = np.array([[0, 0, 0, 0], [1, 7, 6, 6], [1, 3, 2, 5], [0, 5, 6, 0]])
    yp = oracle.conv2d_points(p, Lx, Lx.materialize(xw), Lw, Lw.materialize(ww), pts)
    assert np.array_equal(yp, y[tuple(pts.T)])


def test_epilogue_closed_forms():
    p = _params(1, 4, 5, 5, 6, 3, 3, 1, 1)
    rng = np.random.default_rng(8)
    x = rng.uniform(-1, 1, (1, 4, 5, 5))
    w = rng.uniform(-1, 1, (6, 4, 3, 3))
    s = rng.uniform(0.5, 1.5, 6)
    b = rng.uniform(-0.1, 0.1, 6)
    r = rng.uniform(-1, 1, (1, 6, 5, 5))
    base = oracle.conv2d_f64(p, x, w)
    lin = s[None, :, None, None] * base + b[None, :, None, None] + r
    np.testing.assert_array_equal(oracle.conv2d_f64(p, x, w, s, b, r, 0), lin)
    np.testing.assert_array_equal(oracle.conv2d_f64(p, x, w, s, b, r, 1), np.maximum(lin, 0))
    np.testing.assert_array_equal(oracle.conv2d_f64(p, x, w, s, b, r, 2), np.clip(lin, 0, 6))
    # ReLU of an all-negative pre-activation is all zeros
    neg = oracle.conv2d_f64(p, np.abs(x), -np.abs(w), act=1)
    assert np.all(neg == 0)


def test_gemm_vs_numpy():
    rng = np.random.default_rng(9)
    A = rng.uniform(-1, 1, (37, 53))
    B = rng.uniform(-1, 1, (53, 29))
    np.testing.assert_allclose(oracle.gemm_f64(A, B), A @ B, rtol=1e-12, atol=1e-12)
    bias = rng.uniform(-1, 1, 29)
    np.testing.assert_allclose(oracle.gemm_f64(A, B, bias=bias, act=1),
                               np.maximum(A @ B + bias, 0), rtol=1e-12, atol=1e-12)


def test_gemm_through_tiled_layouts():
    """GEMM template layouts: A M/mt K/kt mt kt, B K/kt N/nt kt nt,
    and NKn (reading A12) read exactly."""
    rng = np.random.default_rng(10)
    M, K, N = 32, 48, 64
    A = rng.uniform(-1, 1, (M, K)).astype(np.float32)
    B = rng.uniform(-1, 1, (K, N)).astype(np.float32)
    La = oracle.Layout((M, K), [("split", 0, [2, 16]), ("split", 2, [3, 16]),
                                ("reorder", [0, 2, 1, 3])])
    Lb = oracle.Layout((K, N), [("split", 0, [3, 16]), ("split", 2, [4, 16]),
                                ("reorder", [0, 2, 1, 3])])
    Lb_nkn = oracle.Layout((K, N), [("split", 1, [4, 16]), ("reorder", [1, 0, 2])])
    want = A.astype(np.float64) @ B.astype(np.float64)
    for lb in (Lb, Lb_nkn):
        got = oracle.gemm(La, La.materialize(A.view(np.uint32)), lb,
                          lb.materialize(B.view(np.uint32)))
        np.testing.assert_allclose(got, want, rtol=1e-12, atol=1e-12)


def test_pool_vs_torch_float64():
    """O9 pooling vs torch max_pool2d / avg_pool2d (count_include_pad=False)."""
    rng = np.random.default_rng(11)
    x = rng.uniform(-1, 1, (2, 5, 13, 11))
    for k, s, p in [(3, 2, 1), (2, 2, 0), (3, 1, 1)]:
        got = oracle.pool2d_f64(x, k, k, s, p, "max")
        ref = torch.nn.functional.max_pool2d(torch.from_numpy(x), k, s, p).numpy()
        assert np.array_equal(got, ref)
        got = oracle.pool2d_f64(x, k, k, s, p, "avg")
        ref = torch.nn.functional.avg_pool2d(torch.from_numpy(x), k, s, p, count_include_pad=False).numpy()
        np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-14)


# ------------------------------------------------------------ dilation (DIL) --
DIL_CASES = [  # (params, dil_h, dil_w): the paper's DIL operator
    (_params(2, 6, 11, 10, 4, 3, 3, 1, 2), 2, 2),
    (_params(1, 4, 13, 9, 3, 3, 2, 2, 1), 3, 2),
    (_params(2, 8, 9, 9, 8, 3, 3, 1, 2, groups=4), 2, 1),
]


def _dil(p, dh, dw):
    q = dict(p)
    q["dil_h"], q["dil_w"] = dh, dw
    return q


@pytest.mark.parametrize("case", DIL_CASES)
def test_dilated_conv_vs_torch_float64(case):
    """O3 with dilation against the library routine (torch float64)"""
    p, dh, dw = case
    q = _dil(p, dh, dw)
    rng = np.random.default_rng(11)
    x = rng.uniform(-1, 1, (p["N"], p["C"], p["H"], p["W"]))
    w = rng.uniform(-1, 1, (p["K"], p["C"] // p["groups"], p["R"], p["S"]))
    y = oracle.conv2d_f64(q, x, w)
    ref = torch.nn.functional.conv2d(torch.from_numpy(x), torch.from_numpy(w), stride=(p["stride_h"], p["stride_w"]),
                                     padding=(p["pad_h"], p["pad_w"]), groups=p["groups"], dilation=(dh, dw)).numpy()
    assert y.shape == ref.shape
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_dilated_conv_brute_force_and_special_cases():
    """bit-exact pure-Python loops (same order); dilation 1 is plain C2D; a
    dilated R x R filter equals the undilated (d(R-1)+1)^2 filter with zeros
    between its taps (the definition of dilation)"""
    p = _params(1, 3, 9, 8, 2, 3, 3, 1, 2)
    rng = np.random.default_rng(12)
    x = rng.uniform(-1, 1, (1, 3, 9, 8))
    w = rng.uniform(-1, 1, (2, 3, 3, 3))
    y = oracle.conv2d_f64(_dil(p, 2, 2), x, w)
    Ho, Wo = (9 + 4 - 4 - 1) // 1 + 1, (8 + 4 - 4 - 1) // 1 + 1
    b = np.zeros((1, 2, Ho, Wo))
    for k, oh, ow in itertools.product(range(2), range(Ho), range(Wo)):
        acc = 0.0
        for c, r, s in itertools.product(range(3), range(3), range(3)):
            ih, iw = oh - 2 + 2 * r, ow - 2 + 2 * s
            if 0 <= ih < 9 and 0 <= iw < 8:
                acc += x[0, c, ih, iw] * w[k, c, r, s]
        b[0, k, oh, ow] = acc
    assert np.array_equal(y, b)
    assert np.array_equal(oracle.conv2d_f64(_dil(p, 1, 1), x, w), oracle.conv2d_f64(p, x, w))
    wz = np.zeros((2, 3, 5, 5))
    wz[:, :, ::2, ::2] = w
    pz = _params(1, 3, 9, 8, 2, 5, 5, 1, 2)
    np.testing.assert_allclose(y, oracle.conv2d_f64(pz, x, wz), rtol=1e-13, atol=1e-13)


def _template(C, H, W, R, V, ht, wt, pad=0):
    """the paper's C2D input template (reading A6) written out
    here (the oracle tests do not import the product's layout helpers)"""
    Bh, Sh, Bw, Sw = V * (ht - 1) + R, V * ht, V * (wt - 1) + R, V * wt
    return [("pad", 2, pad, pad), ("pad", 3, pad, pad), ("unfold", 2, Bh, Sh), ("unfold", 4, Bw, Sw),
            ("split", 1, [C // 8, 8]), ("reorder", [0, 3, 5, 1, 4, 6, 2])]


@pytest.mark.parametrize("H,W,ht,wt", [(12, 12, 2, 2), (13, 9, 2, 4), (16, 10, 4, 1)])
def test_conv_through_lossy_template_reads_only_needed_pixels(H, W, ht, wt):
    """reading A32: a stride-2 1x1 template (windows B = 2(ht - 1) + 1 < S = 2 ht)
    holds only the pixels the conv reads; the oracle's conv through it equals
    torch's conv of the full tensor (the oracle reads the skipped pixels as 0,
    torch sees their real values: equality proves they are never used)"""
    rng = np.random.default_rng(H * 100 + W)
    N, C, K = 2, 16, 8
    x = rng.standard_normal((N, C, H, W))
    w = rng.standard_normal((K, C, 1, 1))
    Lx = oracle.Layout((N, C, H, W), _template(C, H, W, 1, 2, ht, wt))
    assert not Lx.present().all()                 # the template is lossy
    xw = x.astype(np.float32).view(np.uint32)
    phys = Lx.materialize(xw)
    Lw = oracle.Layout((K, C, 1, 1), [])
    ww = w.astype(np.float32).view(np.uint32)
    p = dict(N=N, C=C, H=H, W=W, K=K, R=1, S=1, stride_h=2, stride_w=2, pad_h=0, pad_w=0)
    got = oracle.conv2d(p, Lx, phys, Lw, Lw.materialize(ww))
    ref = torch.nn.functional.conv2d(torch.from_numpy(x.astype(np.float32).astype(np.float64)),
                                     torch.from_numpy(w.astype(np.float32).astype(np.float64)), stride=2).numpy()
    assert np.allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_conv_through_lossy_template_refuses_missing_pixels():
    """the same lossy template under a conv that needs the skipped pixels
    (3x3 stride 1) is refused, never silently read as zeros"""
    N, C, H, W, K = 1, 8, 12, 12, 8
    Lx = oracle.Layout((N, C, H, W), _template(C, H, W, 1, 2, 2, 2))
    phys = Lx.materialize(np.zeros((N, C, H, W), np.uint32))
    Lw = oracle.Layout((K, C, 3, 3), [])
    p = dict(N=N, C=C, H=H, W=W, K=K, R=3, S=3, pad_h=1, pad_w=1)
    with pytest.raises(oracle.OracleError):
        oracle.conv2d(p, Lx, phys, Lw, Lw.materialize(np.zeros((K, C, 3, 3), np.uint32)))
