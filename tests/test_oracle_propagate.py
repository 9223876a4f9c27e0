"""Pins for oracle O7 (Algorithm 1) against the paper's own cases:

  W6/W7  C2D -> ReLU: the ReLU output shares the C2D output layout (Figs. 6-7,
         P:854-919), no conversion;
  W9     C2D -> C2D: one conversion op between them;
  Fig.12 pad -> C2D3x3 -> C2D1x1 has exactly one conversion, between the two
         C2Ds;
  line 10: a simple op between two C2Ds performs the conversion itself (no
         conversion op inserted);
  line 3: non-trivial advanced primitives stop propagation;
  multi-producer rule.
"""
from oracle.propagate import has_nontrivial_advanced, joint_stage, layout_propagation

SHAPE = (1, 64, 56, 56)
NH4WO4 = [("split", 2, [14, 4]), ("reorder", [0, 2, 4, 1, 3])]   # Fig. 6 layout N H/4 W O 4


def test_w6_w7_conv_relu_shares_layout():
    ops = ["complex", "elementwise"]
    edges = [(None, 0, SHAPE, 0), (0, 1, SHAPE, 0), (1, None, SHAPE, 0)]
    P, conv = layout_propagation(ops, edges, 1, NH4WO4, SHAPE)
    assert conv is None
    assert P == {1: NH4WO4, 2: NH4WO4}


def test_w9_conv_conv_inserts_one_conversion():
    ops = ["complex", "complex"]
    edges = [(None, 0, SHAPE, 0), (0, 1, SHAPE, 0), (1, None, SHAPE, 0)]
    P, conv = layout_propagation(ops, edges, 1, NH4WO4, SHAPE)
    assert conv == 1 and P == {1: NH4WO4}


def test_fig12_subgraph_exactly_one_conversion():
    # pad -> C2D 3x3 -> C2D 1x1; each C2D output tuned separately
    s7 = (1, 512, 7, 7)
    ops = ["simple", "complex", "complex"]
    edges = [(None, 0, s7, 0), (0, 1, (1, 512, 9, 9), 0), (1, 2, s7, 0), (2, None, s7, 0)]
    tuned = {2: NH4WO4[:0] + [("split", 1, [64, 8]), ("reorder", [0, 1, 3, 4, 2])],
             3: [("split", 1, [32, 16]), ("reorder", [0, 1, 3, 4, 2])]}
    assign, conversions = joint_stage(ops, edges, tuned, {2: s7, 3: s7})
    assert conversions == {2}
    assert assign[3][0] == 3 and assign[2][0] == 2


def test_line10_simple_op_between_convs_converts_itself():
    ops = ["complex", "elementwise", "complex"]
    edges = [(None, 0, SHAPE, 0), (0, 1, SHAPE, 0), (1, 2, SHAPE, 0), (2, None, SHAPE, 0)]
    P, conv = layout_propagation(ops, edges, 1, NH4WO4, SHAPE)
    assert conv is None           # no conversion op inserted
    assert P == {1: NH4WO4}       # e2 not propagated: the ReLU writes C2D#2's layout


def test_line3_nontrivial_advanced_primitive_stops():
    unf = [("pad", 2, 1, 1), ("unfold", 2, 10, 8)]
    assert has_nontrivial_advanced(unf, SHAPE)
    assert not has_nontrivial_advanced([("pad", 2, 0, 0)], SHAPE)
    assert not has_nontrivial_advanced([("unfold", 2, 8, 8)], SHAPE)   # == split (A9)
    ops = ["complex", "elementwise"]
    edges = [(None, 0, SHAPE, 0), (0, 1, SHAPE, 0), (1, None, SHAPE, 0)]
    P, conv = layout_propagation(ops, edges, 1, unf, SHAPE)
    assert conv == 1 and P == {1: unf}


def test_empty_sequence_is_identity_a21():
    ops = ["complex", "complex"]
    edges = [(None, 0, SHAPE, 0), (0, 1, SHAPE, 0), (1, None, SHAPE, 0)]
    P, conv = layout_propagation(ops, edges, 1, [], SHAPE)
    assert conv is None and P == {1: []}


def test_shape_change_stops_propagation():
    ops = ["complex", "elementwise", "elementwise"]
    small = (1, 64, 28, 28)
    edges = [(None, 0, SHAPE, 0), (0, 1, SHAPE, 0), (1, 2, small, 0), (2, None, small, 0)]
    P, conv = layout_propagation(ops, edges, 1, NH4WO4, SHAPE)
    assert P == {1: NH4WO4}


def test_multi_producer_x0_wins():
    # Y = add(X0, X1): X0 from conv A (slot 0), X1 from conv B (slot 1)
    ops = ["complex", "complex", "elementwise"]
    edges = [(None, 0, SHAPE, 0), (None, 1, SHAPE, 0), (0, 2, SHAPE, 0), (1, 2, SHAPE, 1),
             (2, None, SHAPE, 0)]
    la = [("split", 1, [8, 8]), ("reorder", [0, 1, 3, 4, 2])]
    lb = [("split", 1, [4, 16]), ("reorder", [0, 1, 3, 4, 2])]
    assign, conversions = joint_stage(ops, edges, {2: la, 3: lb}, {2: SHAPE, 3: SHAPE})
    assert assign[4] == (2, la)
    assert conversions == set()
