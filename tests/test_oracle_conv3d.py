"""Pins for oracle O3b, the paper's C3D operator (template
"similar" to C2D):

  * vs torch.nn.functional.conv3d in float64 on CPU (library routine) over
    strides, paddings, dilations and groups;
  * vs a pure-Python 9-loop brute force on a tiny shape (bit-exact: the
    same (c, t, r, s) summation order);
  * special cases: T = 1 equals O3 (conv2d) on every depth slice; a one-hot
    depth tap is O3 on the shifted slice; a 1x1x1 filter equals a GEMM;
  * reading the operands through ALT layouts (NCDHW[x]c, NDHWC, padded and
    unfolded depth) gives bit-identical results (invariant I2, oracle side).
"""
import itertools

import numpy as np
import pytest
import torch

import oracle


def _p(N, C, D, H, W, K, T, R, S, V=(1, 1, 1), pad=(0, 0, 0), dil=(1, 1, 1), groups=1):
    return dict(N=N, C=C, D=D, H=H, W=W, K=K, T=T, R=R, S=S, stride_d=V[0], stride_h=V[1], stride_w=V[2],
                pad_d=pad[0], pad_h=pad[1], pad_w=pad[2], dil_d=dil[0], dil_h=dil[1], dil_w=dil[2], groups=groups)


def _torch(p, x, w):
    return torch.nn.functional.conv3d(
        torch.from_numpy(x), torch.from_numpy(w), stride=(p["stride_d"], p["stride_h"], p["stride_w"]),
        padding=(p["pad_d"], p["pad_h"], p["pad_w"]), dilation=(p["dil_d"], p["dil_h"], p["dil_w"]),
        groups=p["groups"]).numpy()


CASES = [
    _p(2, 8, 6, 7, 7, 16, 3, 3, 3, pad=(1, 1, 1)),                   # C3D-style 3x3x3
    _p(1, 4, 9, 8, 6, 8, 3, 3, 3, V=(2, 2, 1), pad=(1, 1, 1)),       # strided
    _p(2, 3, 5, 9, 9, 8, 3, 7, 7, V=(1, 2, 2), pad=(1, 3, 3)),       # stem-like
    _p(1, 6, 7, 6, 6, 4, 2, 3, 2, dil=(2, 1, 2), pad=(1, 1, 0)),     # dilated
    _p(2, 8, 4, 5, 5, 8, 3, 3, 3, pad=(1, 1, 1), groups=4),          # grouped
    _p(3, 5, 4, 4, 3, 6, 1, 1, 1),                                    # pointwise
]


@pytest.mark.parametrize("p", CASES)
def test_conv3d_vs_torch_float64(p):
    rng = np.random.default_rng(p["C"] * 7 + p["T"])
    x = rng.standard_normal((p["N"], p["C"], p["D"], p["H"], p["W"]))
    w = rng.standard_normal((p["K"], p["C"] // p["groups"], p["T"], p["R"], p["S"]))
    sc, bi = rng.uniform(0.5, 1.5, p["K"]), rng.uniform(-0.1, 0.1, p["K"])
    got = oracle.conv3d_f64(p, x, w, sc, bi, act=0)
    want = _torch(p, x, w) * sc[None, :, None, None, None] + bi[None, :, None, None, None]
    assert got.shape == want.shape
    np.testing.assert_allclose(got, want, rtol=1e-12, atol=1e-12)
    # ReLU6 epilogue with a residual (O6)
    res = rng.standard_normal(want.shape)
    got6 = oracle.conv3d_f64(p, x, w, sc, bi, res, act=2)
    np.testing.assert_allclose(got6, np.clip(want + res, 0.0, 6.0), rtol=1e-12, atol=1e-12)


def test_conv3d_vs_python_brute_force_bit_exact():
    p = _p(1, 2, 3, 4, 3, 2, 2, 2, 3, V=(1, 2, 1), pad=(1, 1, 1))
    rng = np.random.default_rng(3)
    x = rng.standard_normal((1, 2, 3, 4, 3))
    w = rng.standard_normal((2, 2, 2, 2, 3))
    Do, Ho, Wo = oracle.conv3d_out(p)
    want = np.zeros((1, 2, Do, Ho, Wo))
    for n, k, od, oh, ow in itertools.product(range(1), range(2), range(Do), range(Ho), range(Wo)):
        acc = 0.0
        for c, t, r, s in itertools.product(range(2), range(2), range(2), range(3)):
            i_d, i_h, i_w = od - 1 + t, oh * 2 - 1 + r, ow - 1 + s
            if 0 <= i_d < 3 and 0 <= i_h < 4 and 0 <= i_w < 3:
                acc += x[n, c, i_d, i_h, i_w] * w[k, c, t, r, s]
        want[n, k, od, oh, ow] = acc
    assert np.array_equal(oracle.conv3d_f64(p, x, w), want)


def test_conv3d_t1_is_conv2d_per_depth_slice():
    """T = 1 (no depth taps, no depth padding): every output depth slice is O3"""
    p = _p(2, 4, 5, 6, 6, 8, 1, 3, 3, pad=(0, 1, 1))
    rng = np.random.default_rng(5)
    x = rng.standard_normal((2, 4, 5, 6, 6))
    w = rng.standard_normal((8, 4, 1, 3, 3))
    y = oracle.conv3d_f64(p, x, w)
    p2 = dict(N=2, C=4, H=6, W=6, K=8, R=3, S=3, pad_h=1, pad_w=1)
    for d in range(5):
        assert np.array_equal(y[:, :, d], oracle.conv2d_f64(p2, x[:, :, d], w[:, :, 0]))


def test_conv3d_one_hot_depth_tap_is_shifted_conv2d():
    """only depth tap t = 2 non-zero: output depth od reads input depth od + 2 - pd"""
    p = _p(1, 3, 6, 5, 5, 4, 3, 3, 3, pad=(1, 1, 1))
    rng = np.random.default_rng(6)
    x = rng.standard_normal((1, 3, 6, 5, 5))
    w = np.zeros((4, 3, 3, 3, 3))
    w[:, :, 2] = rng.standard_normal((4, 3, 3, 3))
    y = oracle.conv3d_f64(p, x, w)
    p2 = dict(N=1, C=3, H=5, W=5, K=4, R=3, S=3, pad_h=1, pad_w=1)
    for od in range(6):
        i_d = od + 2 - 1
        want = oracle.conv2d_f64(p2, x[:, :, i_d], w[:, :, 2]) if i_d < 6 else np.zeros((1, 4, 5, 5))
        np.testing.assert_allclose(y[:, :, od], want, rtol=1e-13, atol=1e-13)


def test_conv3d_pointwise_is_gemm():
    p = _p(2, 5, 3, 4, 2, 7, 1, 1, 1)
    rng = np.random.default_rng(8)
    x = rng.standard_normal((2, 5, 3, 4, 2))
    w = rng.standard_normal((7, 5, 1, 1, 1))
    want = np.einsum("ncdhw,kc->nkdhw", x, w[:, :, 0, 0, 0])
    np.testing.assert_allclose(oracle.conv3d_f64(p, x, w), want, rtol=1e-13, atol=1e-13)


LAYOUTS_5D = [
    [],
    [("reorder", [0, 2, 3, 4, 1])],                                            # NDHWC
    [("split", 1, [2, 4]), ("reorder", [0, 1, 3, 4, 5, 2])],                  # NCDHW4c
    [("pad", 2, 1, 1), ("split", 1, [1, 8]), ("reorder", [0, 1, 3, 4, 5, 2])],  # depth-padded NCDHW8c
    [("pad", 2, 1, 1), ("unfold", 2, 4, 2), ("split", 1, [1, 8]),
     ("reorder", [0, 2, 1, 3, 4, 5, 6])],                                      # overlapped depth tiles
]


@pytest.mark.parametrize("xi", range(len(LAYOUTS_5D)))
@pytest.mark.parametrize("wi", [0, 1])
def test_conv3d_through_layouts_is_layout_independent(xi, wi):
    p = _p(2, 8, 5, 6, 6, 4, 3, 3, 3, pad=(1, 1, 1))
    rng = np.random.default_rng(11)
    x = (rng.standard_normal((2, 8, 5, 6, 6)).astype(np.float32))
    w = (rng.standard_normal((4, 8, 3, 3, 3)).astype(np.float32))
    want = oracle.conv3d_f64(p, x.astype(np.float64), w.astype(np.float64))
    Lx = oracle.Layout(x.shape, LAYOUTS_5D[xi])
    Lw = oracle.Layout(w.shape, [[], [("reorder", [0, 2, 3, 4, 1])]][wi])
    got = oracle.conv3d(p, Lx, Lx.materialize(x.view(np.uint32)), Lw, Lw.materialize(w.view(np.uint32)))
    assert np.array_equal(got, want)
