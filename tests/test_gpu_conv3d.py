"""GPU parity of alt_conv3d (the paper's C3D; O3b oracle):
the tensor-core path (a depth role in the tcgen05 implicit GEMM: one output
depth slice per M tile, the depth tap moving the TMA box) on channel-tiled
5-D layouts, and the generic CUDA-core path on any layout (fp32 and bf16,
strides, padding, dilation, groups, residual)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth
from tests.helpers import assert_parity, make_operand, read_output

pytestmark = pytest.mark.gpu


def ncdhwxc(C, x, pad_d=0):
    """N C/x D H W x (the 3-D NCHW[x]c), optional materialised depth padding"""
    pr = [("pad", 2, pad_d, pad_d)] if pad_d else []
    return pr + [("split", 1, [C // x, x]), ("reorder", [0, 1, 3, 4, 5, 2])]


def kctrs_yk_xc(K, C, y, x):
    """weights K/y C/x T R S y x (c innermost: K-major B)"""
    return [("split", 0, [K // y, y]), ("split", 2, [C // x, x]), ("reorder", [0, 2, 4, 5, 6, 1, 3])]


NDHWC = [("reorder", [0, 2, 3, 4, 1])]


def run_conv3d(name, N, C, D, H, W, K, T, R, S, V, pad, xp, wp, yp, dtype, dil=(1, 1, 1), groups=1, epi=False,
               res_p=None, act=0, cfg=None, expect_path=None):
    x = synth.activations(name + "x", (N, C, D, H, W))
    w = synth.weights(name + "w", (K, C // groups, T, R, S))
    pd = dict(N=N, C=C, D=D, H=H, W=W, K=K, T=T, R=R, S=S, stride_d=V[0], stride_h=V[1], stride_w=V[2],
              pad_d=pad[0], pad_h=pad[1], pad_w=pad[2], dil_d=dil[0], dil_h=dil[1], dil_w=dil[2], groups=groups)
    out = (N, K) + oracle.conv3d_out(pd)
    Xo, xph, xd = make_operand(name, xp, x, dtype)
    Wo_, wph, wd = make_operand(name, wp, w, dtype)
    p = alt.conv3d_params(N, C, D, H, W, K, T, R, S, V, pad, dil, groups)
    Lx, Lw, Ly = alt.Layout(x.shape, xp), alt.Layout(w.shape, wp), alt.Layout(out, yp)
    y = torch.full(Ly.phys_shape, 3.0, dtype=dtype, device="cuda")  # poison
    kw, ref_kw = {}, {}
    if epi:
        sc, bi = synth.bn_scale(name + "s", K), synth.bn_bias(name + "b", K)
        kw.update(scale=sc.cuda(), bias=bi.cuda())
        ref_kw.update(scale=sc.double().numpy(), bias=bi.double().numpy())
    if res_p is not None:
        r = synth.activations(name + "r", out)
        Ro, rph, rd = make_operand(name + "r", res_p, r, dtype)
        kw.update(residual=rd, residual_l=alt.Layout(out, res_p))
        ref_kw.update(res_l=Ro, residual=rph)
    alt.conv3d(p, Lx, xd, Lw, wd, Ly, y, act=act, cfg=cfg, **kw)
    plan = alt.last_plan()
    torch.cuda.synchronize()
    if expect_path is not None:
        assert plan["path"] == expect_path, plan
    ref = oracle.conv3d(pd, Xo, xph, Wo_, wph, act=act, **ref_kw)
    got = read_output(oracle.Layout(out, yp), y, dtype)
    return assert_parity(got, ref, dtype), plan


TC_CASES = [
    # name, (N, C, D, H, W, K, T, R, S), V, pad, x, w, y, cfg
    ("3x3x3 p1 NCDHW64c", (2, 64, 6, 14, 14, 128, 3, 3, 3), (1, 1, 1), (1, 1, 1), ncdhwxc(64, 64),
     kctrs_yk_xc(128, 64, 128, 64), ncdhwxc(128, 64), {}),
    ("strided depth + hw", (2, 64, 8, 16, 16, 64, 3, 3, 3), (2, 2, 2), (1, 1, 1), ncdhwxc(64, 64),
     kctrs_yk_xc(64, 64, 64, 64), ncdhwxc(64, 64), {"block_n": 64}),
    ("NDHWC in / out, 1x3x3", (3, 32, 5, 12, 12, 64, 1, 3, 3), (1, 1, 1), (0, 1, 1), NDHWC,
     [("reorder", [0, 2, 3, 4, 1])], NDHWC, {}),
    ("depth-padded input, ragged", (2, 32, 5, 9, 11, 48, 3, 3, 3), (1, 1, 1), (1, 1, 1), ncdhwxc(32, 32, pad_d=1),
     kctrs_yk_xc(48, 32, 16, 32), ncdhwxc(48, 16), {"block_n": 64}),
    ("3x1x1 temporal", (2, 64, 8, 7, 7, 128, 3, 1, 1), (1, 1, 1), (1, 0, 0), ncdhwxc(64, 64),
     kctrs_yk_xc(128, 64, 128, 64), ncdhwxc(128, 64), {"cta_pair": 2, "block_n": 128}),
]


@pytest.mark.parametrize("case", TC_CASES, ids=[c[0] for c in TC_CASES])
def test_c3d_tensor_cores(case):
    name, (N, C, D, H, W, K, T, R, S), V, pad, xp, wp, yp, cfg = case
    run_conv3d("c3d" + name, N, C, D, H, W, K, T, R, S, V, pad, xp, wp, yp, torch.bfloat16, epi=True, act=1,
               cfg={"path": alt.PATH_TC, **cfg}, expect_path=alt.PATH_TC)


def test_c3d_auto_takes_tensor_cores():
    _, plan = run_conv3d("c3dauto", 1, 64, 4, 8, 8, 64, 3, 3, 3, (1, 1, 1), (1, 1, 1), ncdhwxc(64, 64),
                         kctrs_yk_xc(64, 64, 64, 64), ncdhwxc(64, 64), torch.bfloat16)
    assert plan["path"] == alt.PATH_TC


SIMT_CASES = [
    # name, (N, C, D, H, W, K, T, R, S), V, pad, dil, groups, x, w, y
    ("NCDHW plain", (2, 4, 5, 6, 6, 8, 3, 3, 3), (1, 1, 1), (1, 1, 1), (1, 1, 1), 1, [], [], []),
    ("strided dilated NDHWC", (1, 8, 9, 8, 7, 4, 3, 2, 3), (2, 1, 2), (1, 0, 1), (2, 1, 1), 1, NDHWC, [], NDHWC),
    ("grouped NCDHW4c", (2, 8, 4, 5, 5, 8, 3, 3, 3), (1, 1, 1), (1, 1, 1), (1, 1, 1), 4, ncdhwxc(8, 4), [],
     ncdhwxc(8, 4)),
    ("stem-like C=3", (2, 3, 5, 9, 9, 8, 3, 7, 7), (1, 2, 2), (1, 3, 3), (1, 1, 1), 1, [], [], ncdhwxc(8, 8)),
]


@pytest.mark.parametrize("dtype", [torch.float32, torch.bfloat16])
@pytest.mark.parametrize("case", SIMT_CASES, ids=[c[0] for c in SIMT_CASES])
def test_c3d_generic_path(case, dtype):
    name, (N, C, D, H, W, K, T, R, S), V, pad, dil, groups, xp, wp, yp = case
    run_conv3d("c3ds" + name, N, C, D, H, W, K, T, R, S, V, pad, xp, wp, yp, dtype, dil=dil, groups=groups,
               epi=True, act=2, cfg={"path": alt.PATH_SIMT}, expect_path=alt.PATH_SIMT)


def test_c3d_residual_falls_back_and_is_exact():
    """a residual (not on the C3D tensor-core path): AUTO serves it exactly
    on the generic path; the output layout is padded (pad zeros written)"""
    _, plan = run_conv3d("c3dres", 2, 16, 4, 6, 6, 16, 3, 3, 3, (1, 1, 1), (1, 1, 1), ncdhwxc(16, 16),
                         kctrs_yk_xc(16, 16, 16, 16), ncdhwxc(16, 8, pad_d=1), torch.bfloat16, epi=True,
                         res_p=NDHWC, act=1)
    assert plan["path"] == alt.PATH_SIMT


def test_c3d_rejects_bad_shapes():
    p = alt.conv3d_params(1, 8, 4, 6, 6, 8, 3, 3, 3, 1, 1)
    Lx = alt.Layout((1, 8, 4, 6, 6), [])
    Lw = alt.Layout((8, 8, 3, 3, 3), [])
    Ly_bad = alt.Layout((1, 8, 4, 6, 7), [])
    x = torch.zeros(Lx.phys_shape, dtype=torch.bfloat16, device="cuda")
    w = torch.zeros(Lw.phys_shape, dtype=torch.bfloat16, device="cuda")
    y = torch.zeros(Ly_bad.phys_shape, dtype=torch.bfloat16, device="cuda")
    with pytest.raises(alt.AltError) as e:
        alt.conv3d(p, Lx, x, Lw, w, Ly_bad, y)
    assert e.value.code == alt._alt.ALT_E_SHAPE


def _divs(n, cands):
    return [c for c in cands if n % c == 0]


@pytest.mark.parametrize("seed", range(120))
def test_c3d_random(seed):
    """random 3-D convs (ragged channels, odd volumes, per-axis stride /
    padding, 1x1x1 .. 3x3x3 windows, NCDHW[x]c / NDHWC layouts, BLOCK_N, CTA
    pair, output-pixel tile) on the tensor cores (bf16), falling back to the
    automatic path where no tensor-core plan exists (and fp32); vs O3b"""
    import random
    rng = random.Random(13000 + seed)
    C, K = 8 * rng.randint(1, 8), 8 * rng.randint(1, 16)
    N, D, H, W = rng.randint(1, 2), rng.randint(2, 7), rng.randint(3, 14), rng.randint(3, 14)
    T, R = rng.choice([1, 3]), rng.choice([1, 3])
    V = tuple(rng.choice([1, 1, 2]) for _ in range(3))
    pad = (rng.randint(0, T // 2), rng.randint(0, R // 2), rng.randint(0, R // 2))
    if (D + 2 * pad[0] - T) < 0 or (H + 2 * pad[1] - R) < 0 or (W + 2 * pad[2] - R) < 0:
        pytest.skip("empty output")
    xc, yc = rng.choice(_divs(C, (8, 16, 32, 64))), rng.choice(_divs(K, (8, 16, 32, 64)))
    xp = rng.choice([ncdhwxc(C, xc), NDHWC])
    wp = rng.choice([kctrs_yk_xc(K, C, rng.choice(_divs(K, (8, 16, 64))), rng.choice(_divs(C, (8, 16, 32)))),
                     [("reorder", [0, 2, 3, 4, 1])]])
    yp = rng.choice([ncdhwxc(K, yc), NDHWC])
    dtype = torch.float32 if rng.random() < 0.15 else torch.bfloat16
    cfg = {"path": alt.PATH_TC, "block_n": rng.choice([64, 128, 256]), "cta_pair": rng.choice([0, 2])}
    if rng.random() < 0.5:
        tw = rng.choice([4, 8, 16, 32])
        th = 128 // tw if 128 // tw <= 32 else 32
        cfg.update(tile_n=1, tile_h=th, tile_w=128 // th)
    act = rng.choice([0, 1])
    if dtype == torch.bfloat16:
        try:
            run_conv3d(f"r3d{seed}", N, C, D, H, W, K, T, R, R, V, pad, xp, wp, yp, dtype, epi=True,
                       act=act, cfg=cfg, expect_path=alt.PATH_TC)
            return
        except alt.AltError as e:
            if e.code != alt._alt.ALT_E_UNSUPPORTED:
                raise
    run_conv3d(f"r3d{seed}", N, C, D, H, W, K, T, R, R, V, pad, xp, wp, yp, dtype, epi=True,
               act=act, cfg={"path": alt.PATH_AUTO})
