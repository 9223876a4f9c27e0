"""Pins for oracle O1/O2 (layout semantics, materialise, relayout).

The oracle is checked against things other than itself:
  * the paper's worked examples W1, W2, W3 (tests/golden/, with citations);
  * numpy library routines (reshape / transpose / pad /
    sliding_window_view) applied to an array of logical indices, which
    brute-forces G on every physical position of random tiny layouts;
  * the closed form T = ceil((D-B)/S) + 1 of the unfolded extent;
  * invariants: relayout round trip (I1) and composition.
"""
import os
import random

import numpy as np
import pytest

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ------------------------------------------------------------------ W1-W3 --
def _golden_rows(name):
    rows = []
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if line and not line.startswith("#"):
            rows.append(line)
    return rows


def test_w1_split_reorder_shape_and_values():
    for row in _golden_rows("w1_w2_shapes.txt"):
        case, rest = row.split(None, 1)
        if case != "W1":
            continue
        spec, want = rest.split(";")
        N, O, H, W, ot = map(int, spec.split())
        want = tuple(map(int, want.split()))
        # paper: split(dim=2, [O//ot, ot]); reorder([1,2,4,5,3]) (1-based, A1)
        L = oracle.Layout((N, O, H, W), [("split", 1, [O // ot, ot]),
                                         ("reorder", [0, 1, 3, 4, 2])])
        assert L.phys_shape == want
        x = np.arange(N * O * H * W, dtype=np.uint32).reshape(N, O, H, W)
        ref = x.reshape(N, O // ot, ot, H, W).transpose(0, 1, 3, 4, 2)
        assert np.array_equal(L.materialize(x), ref)


def test_w2_fuse_split_reorder_access_expression():
    for row in _golden_rows("w1_w2_shapes.txt"):
        case, rest = row.split(None, 1)
        if case != "W2":
            continue
        spec, want = rest.split(";")
        N, O, H, W, _ = map(int, spec.split())
        want = tuple(map(int, want.split()))
        L = oracle.Layout((N, H, W, O), [("fuse", 1, 3),
                                         ("split", 1, [O // 4, 4, H * W]),
                                         ("reorder", [0, 1, 3, 2])])
        assert L.phys_shape == want
        for n in range(N):
            for h in range(H):
                for w in range(W):
                    for o in range(O):
                        e = h * (W * O) + w * O + o          # step 1 of P:712-716
                        paper = (n, e // (H * W * 4), e % (H * W), (e // (H * W)) % 4)
                        assert L.F((n, h, w, o)) == paper
                        assert L.G(paper) == (n, h, w, o)


def test_w3_unfold_golden():
    rows = _golden_rows("unfold_w3.txt")
    D, B, S = map(int, rows[0].split())
    inp = np.array(list(map(int, rows[1].split())), np.uint32)
    want = np.array([list(map(int, r.split())) for r in rows[2:]], np.uint32)
    L = oracle.Layout((D,), [("unfold", 0, B, S)])
    assert L.phys_shape == want.shape
    assert np.array_equal(L.materialize(inp), want)


@pytest.mark.parametrize("D,B,S", [(5, 3, 2), (230, 13, 8), (58, 10, 8), (7, 7, 1),
                                   (9, 2, 3), (16, 4, 4), (1, 1, 1), (10, 3, 5)])
def test_unfold_extent_closed_form(D, B, S):
    L = oracle.Layout((D,), [("unfold", 0, B, S)])
    T = -(-(D - B) // S) + 1
    assert L.phys_shape == (T, B)


def test_unfold_r18_conv1_table3_reading_a3():
    # Table 3 searched layout ht = 4 on the padded 230 input,
    # stride 2, 7x7: S = V*ht = 8, B = V(ht-1)+R = 13 (reading A6) -> T = 29
    # while the conv needs ceil(112/4) = 28 tiles (reading A3: extra tile is
    # dead overhang).
    L = oracle.Layout((230,), [("unfold", 0, 13, 8)])
    assert L.phys_shape == (29, 13)
    assert -(-112 // 4) == 28


def test_unfold_bad_args():
    with pytest.raises(oracle.OracleError) as ei:
        oracle.Layout((4,), [("unfold", 0, 5, 1)])
    assert ei.value.code == oracle.E_SHAPE
    with pytest.raises(oracle.OracleError) as ei:
        oracle.Layout((6,), [("split", 0, [4, 2])])
    assert ei.value.code == oracle.E_NONDIV


# ---------------------------------------------------- numpy brute force --
def np_apply(idx: np.ndarray, prims):
    """Independent reference: apply the primitives with numpy routines to an
    array of logical linear indices (-1 marks structural zeros)."""
    a = idx
    for p in prims:
        k = p[0]
        if k == "split":
            d, f = p[1], p[2]
            a = a.reshape(a.shape[:d] + tuple(f) + a.shape[d + 1:])
        elif k == "reorder":
            a = a.transpose(p[1])
        elif k == "fuse":
            d, m = p[1], p[2]
            a = a.reshape(a.shape[:d] + (int(np.prod(a.shape[d:d + m])),) + a.shape[d + m:])
        elif k == "pad":
            d, lo, hi = p[1:]
            pw = [(0, 0)] * a.ndim
            pw[d] = (lo, hi)
            a = np.pad(a, pw, constant_values=-1)
        elif k == "unfold":
            d, B, S = p[1:]
            D = a.shape[d]
            T = -(-(D - B) // S) + 1
            need = (T - 1) * S + B
            pw = [(0, 0)] * a.ndim
            pw[d] = (0, need - D)
            a = np.pad(a, pw, constant_values=-1)
            win = np.lib.stride_tricks.sliding_window_view(a, B, axis=d)[
                (slice(None),) * d + (slice(None, None, S),)]
            a = np.moveaxis(win, -1, d + 1).copy()
    return a


def random_prims(shape, rng, n=4):
    shape = list(shape)
    prims = []
    for _ in range(n):
        r = len(shape)
        kind = rng.choice(["split", "reorder", "fuse", "pad", "unfold"])
        d = rng.randrange(r)
        if kind == "split":
            divs = [f for f in range(1, shape[d] + 1) if shape[d] % f == 0]
            f = rng.choice(divs)
            if len(shape) + 1 > 8:
                continue
            prims.append(("split", d, [shape[d] // f, f]))
            shape = shape[:d] + [shape[d] // f, f] + shape[d + 1:]
        elif kind == "reorder":
            perm = list(range(r))
            rng.shuffle(perm)
            prims.append(("reorder", perm))
            shape = [shape[i] for i in perm]
        elif kind == "fuse":
            if r < 2:
                continue
            d = rng.randrange(r - 1)
            m = rng.randint(2, min(3, r - d))
            prod = int(np.prod(shape[d:d + m]))
            if prod > 64:
                continue
            prims.append(("fuse", d, m))
            shape = shape[:d] + [prod] + shape[d + m:]
        elif kind == "pad":
            lo, hi = rng.randint(0, 2), rng.randint(0, 2)
            prims.append(("pad", d, lo, hi))
            shape[d] += lo + hi
        elif kind == "unfold":
            if len(shape) + 1 > 8:
                continue
            B = rng.randint(1, shape[d])
            S = rng.randint(1, B + 1)
            T = -(-(shape[d] - B) // S) + 1
            prims.append(("unfold", d, B, S))
            shape = shape[:d] + [T, B] + shape[d + 1:]
    return prims


@pytest.mark.parametrize("seed", range(60))
def test_G_and_F_bruteforce_vs_numpy(seed):
    rng = random.Random(seed)
    rank = rng.randint(1, 4)
    shape = tuple(rng.randint(1, 6) for _ in range(rank))
    prims = random_prims(shape, rng, n=rng.randint(1, 5))
    L = oracle.Layout(shape, prims)
    n = int(np.prod(shape))
    ref = np_apply(np.arange(n, dtype=np.int64).reshape(shape), prims)
    assert L.phys_shape == ref.shape
    flat = ref.reshape(-1)
    for j in range(flat.size):
        g = L.G_linear(j)
        if flat[j] < 0:
            assert g is None
        else:
            assert g is not None and int(np.ravel_multi_index(g, shape)) == flat[j]
    # F lands on a position that holds the element (owner copy), or the
    # element truly has no copy (lossy)
    held = set(flat[flat >= 0].tolist())
    for i in range(n):
        li = np.unravel_index(i, shape)
        jf = L.F_linear(li)
        if i in held:
            assert jf >= 0 and flat[jf] == i
        else:
            assert jf < 0
    # materialise == numpy gather
    x = (np.arange(n, dtype=np.uint32) * 7 + 3).reshape(shape)
    want = np.where(ref >= 0, x.reshape(-1)[np.maximum(ref, 0)], 0).astype(np.uint32)
    assert np.array_equal(L.materialize(x), want)
    assert L.check_consistent(want) == 0
    # unmaterialise (O2, F side) == numpy scatter of the owner copies: every
    # held element reads back from the numpy image, a lossy layout is refused
    if len(held) == n:
        assert np.array_equal(L.unmaterialize(want), x)
    else:
        with pytest.raises(oracle.OracleError):
            L.unmaterialize(want)


def test_pad_matches_numpy_pad():
    x = np.arange(2 * 3 * 4, dtype=np.uint16).reshape(2, 3, 4) + 1
    L = oracle.Layout(x.shape, [("pad", 1, 2, 1), ("pad", 2, 0, 3)])
    assert np.array_equal(L.materialize(x), np.pad(x, [(0, 0), (2, 1), (0, 3)]))


def test_consistency_checker_detects_corruption():
    x = np.arange(1, 13, dtype=np.uint32).reshape(3, 4)
    L = oracle.Layout(x.shape, [("pad", 0, 1, 1), ("unfold", 1, 3, 1)])
    P = L.materialize(x)
    assert L.check_consistent(P) == 0
    Q = P.copy()
    Q[0, 0, 0] = 5              # a pad position must be zero
    assert L.check_consistent(Q) == 1
    Q = P.copy()
    Q[1, 1, 0] = 99             # second copy of x[0,1] differs from the owner
    assert L.check_consistent(Q) >= 1


# ------------------------------------------------------------ relayout --
LAYOUTS_NCHW = [
    [],
    [("reorder", [0, 2, 3, 1])],                                     # NHWC
    [("split", 1, [4, 4]), ("reorder", [0, 1, 3, 4, 2])],           # NCHW4c
    [("split", 1, [2, 8]), ("reorder", [0, 1, 3, 4, 2])],           # NCHW8c
    [("pad", 2, 1, 1), ("pad", 3, 1, 1), ("unfold", 2, 9, 7),
     ("unfold", 4, 9, 7), ("split", 1, [2, 8]),
     ("reorder", [0, 3, 5, 1, 4, 6, 2])],                            # tiled, Fig. 2
    [("fuse", 1, 3), ("split", 1, [4, 4, 196]), ("reorder", [0, 1, 3, 2])],  # W2-like
]


@pytest.mark.parametrize("a", range(len(LAYOUTS_NCHW)))
@pytest.mark.parametrize("b", range(len(LAYOUTS_NCHW)))
def test_relayout_roundtrip_and_composition(a, b):
    shape = (2, 16, 14, 14)
    rng = np.random.default_rng(a * 10 + b)
    x = rng.integers(0, 2**16, size=shape, dtype=np.uint16)   # random bit patterns
    La = oracle.Layout(shape, LAYOUTS_NCHW[a])
    Lb = oracle.Layout(shape, LAYOUTS_NCHW[b])
    L0 = oracle.Layout(shape, [])
    xa = La.materialize(x)
    xb = oracle.relayout(La, xa, Lb)
    assert np.array_equal(xb, Lb.materialize(x))                  # composition
    assert np.array_equal(oracle.relayout(Lb, xb, La), xa)        # I1 round trip
    assert np.array_equal(oracle.relayout(Lb, xb, L0), x)


def test_relayout_lossy_source_rejected():
    x = np.arange(10, dtype=np.uint32)
    gap = oracle.Layout((10,), [("unfold", 0, 2, 3)])              # B < S: gaps
    ident = oracle.Layout((10,), [])
    with pytest.raises(oracle.OracleError) as ei:
        oracle.relayout(gap, gap.materialize(x), ident)
    assert ei.value.code == oracle.E_LOSSY
