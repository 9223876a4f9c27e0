"""CPU-side tests of the product boundary (no GPU needed):

  * libalt.so loads and exports every symbol include/alt.h declares;
  * the layout compiler (alt_layout_create + the host-only map queries)
    agrees with the oracle's G / F on every physical position of random
    layouts and on the paper's examples;
  * flags (lossless / pad / unfold / separable / identity);
  * error codes for bad primitive sequences;
  * alt_plan_chain (Alg. 1) agrees with the oracle's propagate.py;
  * compute calls reject host pointers (no CPU fallback).
"""
import os
import random
import re

import numpy as np
import pytest
import torch

import oracle
from oracle.propagate import joint_stage
import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import _alt
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import layouts as LY
from tests.test_oracle_layout import LAYOUTS_NCHW, random_prims

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "alt.h")).read()
    declared = set(re.findall(r"\b(alt_[a-z0-9_]+)\s*\(", hdr))
    declared = {d for d in declared if not d.endswith("_t")}
    assert declared == set(_alt.EXPORTED), declared ^ set(_alt.EXPORTED)
    for name in declared:
        assert hasattr(_alt._lib, name), name


def _compare_with_oracle(shape, prims):
    P = alt.Layout(shape, prims)
    O = oracle.Layout(shape, prims)
    assert P.phys_shape == O.phys_shape
    for j in range(P.phys_numel):
        assert P.phys_to_logical(j) == O.G_linear(j), (j, prims)
    for i in range(int(np.prod(shape))):
        li = tuple(int(v) for v in np.unravel_index(i, shape))
        jo = O.F_linear(li)
        jp = P.logical_to_phys(li)
        assert (jp if jp is not None else -1) == jo, (li, prims)
    return P, O


@pytest.mark.parametrize("seed", range(80))
def test_layout_compiler_matches_oracle_random(seed):
    rng = random.Random(1000 + seed)
    rank = rng.randint(1, 4)
    shape = tuple(rng.randint(1, 6) for _ in range(rank))
    prims = random_prims(shape, rng, n=rng.randint(1, 5))
    _compare_with_oracle(shape, prims)


@pytest.mark.parametrize("i", range(len(LAYOUTS_NCHW)))
def test_layout_compiler_matches_oracle_nchw_family(i):
    P, _ = _compare_with_oracle((2, 16, 14, 14), LAYOUTS_NCHW[i])
    if i in (0, 1, 2, 3):
        assert P.lossless and P.separable
    if i == 0:
        assert P.identity
    if i == 4:
        assert P.flags & _alt.ALT_HAS_PAD and P.flags & _alt.ALT_HAS_UNFOLD and P.separable
    if i == 5:
        assert not P.separable


def test_flags_and_errors():
    L = alt.Layout((10,), [("unfold", 0, 2, 3)])
    assert not L.lossless
    with pytest.raises(alt.AltError) as e:
        alt.Layout((6,), [("split", 0, [4, 2])])
    assert e.value.code == _alt.ALT_E_NONDIVISIBLE
    with pytest.raises(alt.AltError) as e:
        alt.Layout((4,), [("unfold", 0, 5, 1)])
    assert e.value.code == _alt.ALT_E_SHAPE
    with pytest.raises(alt.AltError) as e:
        alt.Layout((4, 4), [("reorder", [0, 0])])
    assert e.value.code == _alt.ALT_E_INVALID
    # templates from layouts.py are valid, separable and lossless
    for prims in (LY.nchwxc(64, 16), LY.nchwxc(3, 8, pad_c=5), LY.kcrs_yk_xc(64, 64, 16, 16),
                  LY.kcrs_paper(64, 64, 16, 16)):
        shape = (64, 64, 3, 3) if prims[0][0] != "pad" and "kcrs" else None
    Lx = alt.Layout((2, 3, 8, 8), LY.nchwxc(3, 8, pad_c=5))
    assert Lx.phys_shape == (2, 1, 8, 8, 8) and Lx.flags & _alt.ALT_HAS_PAD
    Lw = alt.Layout((64, 64, 3, 3), LY.kcrs_yk_xc(64, 64, 16, 16))
    assert Lw.phys_shape == (4, 4, 3, 3, 16, 16) and Lw.lossless
    Lt = alt.Layout((1, 64, 56, 56), LY.conv_input_tiled(64, 16, 56, 56, 3, 3, 8, 8, 1, 1))
    assert Lt.phys_shape == (1, 7, 7, 4, 10, 10, 16)


def test_compute_calls_reject_host_pointers():
    L = alt.Layout((4, 4), [])
    a = torch.zeros(4, 4)
    with pytest.raises(alt.AltError) as e:
        alt.relayout(L, a, L, torch.zeros(4, 4), stream=_FakeStream())
    assert e.value.code == _alt.ALT_E_INVALID


class _FakeStream:
    cuda_stream = 0


def _plan_case(ops_kinds, edges, tuned):
    """Run both the product (alt_plan_chain) and the oracle on one graph."""
    kind_code = {"complex": 0, "elementwise": 1, "simple": 2}
    shapes = {e: edges[e][2] for e in range(len(edges))}
    lay = []
    for e, (s, d, shp, slot) in enumerate(edges):
        lay.append(alt.Layout(shp, tuned[e]) if e in tuned else None)
    src, conv = alt.plan_chain([kind_code[k] for k in ops_kinds],
                               [(s if s is not None else -1, d if d is not None else -1, slot,
                                 int(np.prod(shp))) for (s, d, shp, slot) in edges], lay)
    assign, conversions = joint_stage(ops_kinds, edges, tuned, shapes)
    want_src = [assign[e][0] if e in assign else -1 for e in range(len(edges))]
    # the oracle records tuned edges as their own source
    assert src == want_src, (src, want_src)
    assert {e for e, c in enumerate(conv) if c} == conversions


def test_plan_chain_matches_oracle():
    S = (1, 64, 56, 56)
    t1 = [("split", 1, [8, 8]), ("reorder", [0, 1, 3, 4, 2])]
    t2 = [("split", 1, [4, 16]), ("reorder", [0, 1, 3, 4, 2])]
    # conv -> relu -> out
    _plan_case(["complex", "elementwise"], [(None, 0, S, 0), (0, 1, S, 0), (1, None, S, 0)], {1: t1})
    # conv -> conv
    _plan_case(["complex", "complex"], [(None, 0, S, 0), (0, 1, S, 0), (1, None, S, 0)], {1: t1, 2: t2})
    # conv -> relu -> conv (ReLU converts)
    _plan_case(["complex", "elementwise", "complex"],
               [(None, 0, S, 0), (0, 1, S, 0), (1, 2, S, 0), (2, None, S, 0)], {1: t1, 3: t2})
    # residual block: conv a, conv b -> add (X0 wins) -> relu -> out
    _plan_case(["complex", "complex", "elementwise", "elementwise"],
               [(None, 0, S, 0), (None, 1, S, 0), (0, 2, S, 0), (1, 2, S, 1), (2, 3, S, 0),
                (3, None, S, 0)], {2: t1, 3: t2})
    # non-trivial advanced primitive stops propagation with a conversion
    unf = [("pad", 2, 1, 1), ("unfold", 2, 10, 8)]
    _plan_case(["complex", "elementwise"], [(None, 0, S, 0), (0, 1, S, 0), (1, None, S, 0)], {1: unf})


def test_zero_extent_layouts_are_rejected():
    """a layout needs every logical extent >= 1 (empty batches are handled
    by the operators themselves: N = 0 / M = 0 calls are no-ops)"""
    import paper_conf_eurosys_xuxpwwwdxcwc23_b200 as alt
    for shp in [(0, 16, 4, 4), (5, 0)]:
        with pytest.raises(alt.AltError) as e:
            alt.Layout(shp, [])
        assert e.value.code == alt._alt.ALT_E_INVALID


def test_store_at_argument_errors_without_gpu():
    """alt_store_at / alt_decouple_at / alt_matmul_store_at validate shapes,
    dims, dtypes and the epilogue before touching any pointer (no GPU)."""
    La, Lz, Lbad = alt.Layout((8, 4), []), alt.Layout((9, 4), []), alt.Layout((8, 5), [])
    L = _alt._lib
    codes = {
        "null layout": L.alt_store_at(None, None, None, 0, Lz.handle, None, alt.ALT_BF16, None),
        "dim range": L.alt_store_at(La.handle, None, None, 2, Lz.handle, None, alt.ALT_BF16, None),
        "bad dtype": L.alt_store_at(La.handle, None, None, 0, Lz.handle, None, 9, None),
        "wrong dim": L.alt_store_at(La.handle, None, None, 1, Lz.handle, None, alt.ALT_BF16, None),
        "decouple shape": L.alt_decouple_at(Lz.handle, None, 0, Lbad.handle, None, None, alt.ALT_F32, None),
        "gemm z shape": L.alt_matmul_store_at(16, 4, 9, alt.Layout((16, 9), []).handle, None, Lz.handle,
                                              None, alt.Layout((16, 4), []).handle, None, alt.ALT_BF16,
                                              None, None, None),
        "host pointers": L.alt_store_at(La.handle, np.zeros(32, np.uint16).ctypes.data, np.zeros(4, np.uint16).ctypes.data,
                                        0, Lz.handle, np.zeros(36, np.uint16).ctypes.data, alt.ALT_BF16, None),
    }
    E_INVALID, E_SHAPE = 1, 2
    assert codes["null layout"] == E_INVALID
    assert codes["dim range"] == E_INVALID
    assert codes["bad dtype"] == E_INVALID
    assert codes["wrong dim"] == E_SHAPE
    assert codes["decouple shape"] == E_SHAPE
    assert codes["gemm z shape"] == E_SHAPE
    assert codes["host pointers"] == E_INVALID


@pytest.mark.parametrize("seed", range(150))
def test_plan_chain_random_dags_match_oracle(seed):
    """random op DAGs (complex / elementwise ops, chains with skip edges and
    two-input elementwise adds, several outputs) with random tuned output
    layouts on the complex ops (tiled channels, a non-trivial pad + unfold):
    alt_plan_chain (Alg. 1 + the multi-producer rule, plan.cpp) against the
    oracle's joint stage (O7) edge by edge"""
    rng = random.Random(17000 + seed)
    S = (1, 64, 28, 28)
    lays = [[("split", 1, [8, 8]), ("reorder", [0, 1, 3, 4, 2])],
            [("split", 1, [4, 16]), ("reorder", [0, 1, 3, 4, 2])],
            [("pad", 2, 1, 1), ("unfold", 2, 10, 8)],
            [("reorder", [0, 2, 3, 1])]]
    n = rng.randint(2, 7)
    kinds = [rng.choice(["complex", "elementwise"]) for _ in range(n)]
    edges = [(None, 0, S, 0)]
    used = set()  # a complex op's output tensor has one tuned layout: one consumer edge
    def pick(i, exclude=()):
        cand = [j for j in range(i) if j not in exclude and not (kinds[j] == "complex" and j in used)]
        if not cand:
            return None
        j = i - 1 if (i - 1 in cand and rng.random() < 0.7) else rng.choice(cand)
        used.add(j)
        return j
    for i in range(1, n):
        src = pick(i)
        edges.append((src, i, S, 0))
        if kinds[i] == "elementwise" and i >= 2 and rng.random() < 0.4:
            src2 = pick(i, exclude=(src,))
            if src2 is not None:
                edges.append((src2, i, S, 1))
    consumed = {s for (s, d, _, _) in edges if s is not None}
    for i in range(n):
        if i not in consumed or (kinds[i] != "complex" and rng.random() < 0.15):
            edges.append((i, None, S, 0))
    tuned = {}
    for e, (s, d, _, _) in enumerate(edges):
        if s is not None and kinds[s] == "complex" and rng.random() < 0.8:
            tuned[e] = rng.choice(lays)
    if not tuned:
        pytest.skip("no tuned layout")
    _plan_case(kinds, edges, tuned)
