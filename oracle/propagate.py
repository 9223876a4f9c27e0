"""O7 — Algorithm 1 "Layout Propagation" (§4.2) step by step.
TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Graph: ``ops[i]`` is "complex" (C2D, GMM: tuned), "elementwise"
(Y[i] = F(X[i])) or "simple" (any other op, e.g. pad / pool: a
conversion boundary, reading A10).  ``edges[e] = (src_op, dst_op, shape,
in_idx)``; src_op None = graph input, dst_op None = graph output; in_idx is
the input slot of the tensor at dst_op.

``layout_propagation(ops, edges, e_T, p_T)`` follows the algorithm line by
line and returns ``(P, conversion)`` where P maps edge -> primitive sequence
and ``conversion`` is the edge before whose consumer a conversion op is
inserted (or None).

Readings: A9 "non-trivial advanced primitive", A21 (p_T empty
means no layout change, so the conversion is the identity and is elided).
"""
from __future__ import annotations

from collections import deque


def is_trivial_advanced(prim, shape_before_dim: int | None = None) -> bool:
    """A9: pad with lo = hi = 0, or unfold with B = D and one tile, or unfold
    with B = S dividing D (== split), is trivial."""
    kind = prim[0]
    if kind == "pad":
        return prim[2] == 0 and prim[3] == 0
    if kind == "unfold":
        B, S = prim[2], prim[3]
        if shape_before_dim is not None and B == shape_before_dim:
            return True
        return B == S and shape_before_dim is not None and shape_before_dim % S == 0
    return True  # split / reorder / fuse are basic primitives


def has_nontrivial_advanced(prims, logical_shape) -> bool:
    shape = list(logical_shape)
    for p in prims:
        k = p[0]
        d = p[1] if k != "reorder" else None
        if k in ("pad", "unfold") and not is_trivial_advanced(p, shape[d]):
            return True
        # advance the shape (needed for the next primitive's extent)
        if k == "split":
            shape = shape[:d] + list(p[2]) + shape[d + 1:]
        elif k == "reorder":
            shape = [shape[i] for i in p[1]]
        elif k == "fuse":
            prod = 1
            for x in shape[d:d + p[2]]:
                prod *= x
            shape = shape[:d] + [prod] + shape[d + p[2]:]
        elif k == "unfold":
            B, S = p[2], p[3]
            T = -(-(shape[d] - B) // S) + 1
            shape = shape[:d] + [T, B] + shape[d + 1:]
        elif k == "pad":
            shape[d] = shape[d] + p[2] + p[3]
    return False


def layout_propagation(ops, edges, e_T: int, p_T, logical_shape):
    """Algorithm 1.  Returns (P, conversion_edge or None)."""
    P = {e_T: list(p_T)}                                     # line 2
    o1, o2, _, _ = edges[e_T]
    if (not p_T or has_nontrivial_advanced(p_T, logical_shape)
            or (o2 is not None and ops[o2] == "complex")):   # line 3
        conv = e_T if (p_T and o2 is not None) else None     # line 4 (A21)
        return P, conv                                       # line 5
    Q = deque([e_T])                                         # line 6
    while Q:                                                 # line 7
        s = Q.popleft()                                      # line 8
        _, s_o2, s_shape, _ = edges[s]
        for t, (t_o2, t_o3, t_shape, _) in enumerate(edges):  # line 9
            if t_o2 is None or t_o2 != s_o2:
                continue
            if (ops[s_o2] == "elementwise" and tuple(t_shape) == tuple(s_shape)
                    and (t_o3 is None or ops[t_o3] != "complex")):  # line 10
                P[t] = list(P[s])                            # line 11
                Q.append(t)                                  # line 12
    return P, None                                           # line 13


def joint_stage(ops, edges, tuned_layouts: dict, logical_shapes: dict):
    """§6: every complex op's tuned output layout is propagated
    with Algorithm 1 (``layout_propagation``, verbatim); where several tuned
    layouts reach the same tensor, the multi-producer rule decides: the
    layout that enters the elementwise producer through its lowest input slot
    (X0) wins.  Reading A31: the slot is judged by the layout each input
    tensor finally carries — inputs are settled before outputs, in
    topological order — so a layout that lost at an upstream elementwise op
    does not enter downstream ops through that op's output.

    tuned_layouts: edge -> primitive sequence of each complex op's output.
    Returns (assign: edge -> (source edge, prims), conversions: set of edges).
    """
    reach: dict[int, dict] = {}   # tuned edge -> {edge: prims} (Alg. 1's P)
    conversions = set()
    for e_T in sorted(tuned_layouts):
        P, conv = layout_propagation(ops, edges, e_T, tuned_layouts[e_T], logical_shapes[e_T])
        if conv is not None:
            conversions.add(conv)
        reach[e_T] = P
    assign: dict[int, tuple[int, list]] = {}
    for e in _topological_edges(ops, edges):
        if e in tuned_layouts:                   # a tuned tensor keeps its own layout
            assign[e] = (e, list(tuned_layouts[e]))
            continue
        cands = [T for T in reach if e in reach[T]]
        if not cands:
            continue
        producer = edges[e][0]
        inputs = sorted((edges[i][3], i) for i in range(len(edges)) if edges[i][1] == producer)
        for _, i in inputs:                      # X0: the lowest slot carrying a candidate
            if i in assign and assign[i][0] in cands:
                T = assign[i][0]
                assign[e] = (T, reach[T][e])
                break
    return assign, conversions


def _topological_edges(ops, edges):
    """Edges ordered so that every input edge of an op precedes its output
    edges (Kahn's algorithm over the ops; graph inputs first)."""
    n = len(ops)
    indeg = [0] * n
    for a, b, _, _ in edges:
        if a is not None and b is not None:
            indeg[b] += 1
    order, ready = [], [o for o in range(n) if indeg[o] == 0]
    while ready:
        o = ready.pop(0)
        order.append(o)
        for a, b, _, _ in edges:
            if a == o and b is not None:
                indeg[b] -= 1
                if indeg[b] == 0:
                    ready.append(b)
    rank = {o: k for k, o in enumerate(order)}
    return sorted(range(len(edges)), key=lambda e: (-1 if edges[e][0] is None else rank[edges[e][0]], e))
