"""Builders for the layout families of ALT's tuning templates (§5.1,
P:1092-1179).  Plain primitive sequences (0-based dims, reading A1)."""
from __future__ import annotations


def nchw():
    return []


def nhwc():
    return [("reorder", [0, 2, 3, 1])]


def nchwxc(C: int, x: int, pad_c: int = 0, pad_hw: int = 0):
    """N C/x H W x (the paper's N O/ot H W ot).  pad_c zeros are
    appended to C first when x does not divide C (reading A2); pad_hw
    materialises conv zero padding on H and W (A7)."""
    pr = []
    if pad_c:
        pr.append(("pad", 1, 0, pad_c))
    if pad_hw:
        pr += [("pad", 2, pad_hw, pad_hw), ("pad", 3, pad_hw, pad_hw)]
    Cp = C + pad_c
    pr += [("split", 1, [Cp // x, x]), ("reorder", [0, 1, 3, 4, 2])]
    return pr


def kcrs_yk_xc(K: int, C: int, y: int, x: int, pad_c: int = 0):
    """Weights K/y C/x R S y x (c innermost: K-major B operand, reading A11)."""
    pr = []
    if pad_c:
        pr.append(("pad", 1, 0, pad_c))
    Cp = C + pad_c
    pr += [("split", 0, [K // y, y]), ("split", 2, [Cp // x, x]),
           ("reorder", [0, 2, 4, 5, 1, 3])]
    return pr


def kcrs_paper(K: int, C: int, ot: int, it: int):
    """The paper's weight template O/o't I/i't KH KW i't o't."""
    return [("split", 0, [K // ot, ot]), ("split", 2, [C // it, it]),
            ("reorder", [0, 2, 4, 5, 3, 1])]


def conv_input_tiled(C: int, it: int, H: int, W: int, R: int, S: int, ht: int, wt: int,
                     stride: int = 1, pad: int = 0):
    """The paper's C2D input template N H/ht W/wt I/it (ht+KH-1)(wt+KW-1) it
     with pad before unfold; stride V uses S = V ht,
    B = V(ht-1)+R (reading A6)."""
    V = stride
    Bh, Sh = V * (ht - 1) + R, V * ht
    Bw, Sw = V * (wt - 1) + S, V * wt
    return [("pad", 2, pad, pad), ("pad", 3, pad, pad), ("unfold", 2, Bh, Sh),
            ("unfold", 4, Bw, Sw), ("split", 1, [C // it, it]),
            ("reorder", [0, 3, 5, 1, 4, 6, 2])]


def conv_output_tiled(K: int, ot: int, Ho: int, Wo: int, ht: int, wt: int):
    """Output template N H/ht W/wt O/ot ht wt ot."""
    return [("split", 2, [Ho // ht, ht]), ("split", 4, [Wo // wt, wt]),
            ("split", 1, [K // ot, ot]), ("reorder", [0, 3, 5, 1, 4, 6, 2])]


def gemm_a_tiled(M: int, K: int, mt: int, kt: int):
    """A: M/mt K/kt mt kt."""
    return [("split", 0, [M // mt, mt]), ("split", 2, [K // kt, kt]), ("reorder", [0, 2, 1, 3])]


def gemm_b_tiled_nk(K: int, N: int, nt: int, kt: int):
    """B stored N/nt K/kt nt kt (K innermost: K-major B operand)."""
    return [("split", 0, [K // kt, kt]), ("split", 2, [N // nt, nt]), ("reorder", [2, 0, 3, 1])]


def gemm_z_tiled_nk(K: int, N: int, nt: int, kt: int):
    """Z = store_at(B, bias, 0), logical [K + 1, N], stored like
    gemm_b_tiled_nk with one more K tile: N/nt (K+kt)/kt nt kt, K a multiple
    of kt; the bias row k = K opens the last K tile (pad zeros after it)."""
    return [("pad", 0, 0, kt - 1), ("split", 0, [(K + kt) // kt, kt]), ("split", 2, [N // nt, nt]),
            ("reorder", [2, 0, 3, 1])]


def gemm_b_tiled_kn(K: int, N: int, kt: int, nt: int):
    """B: K/kt N/nt kt nt (the paper's template; N innermost)."""
    return [("split", 0, [K // kt, kt]), ("split", 2, [N // nt, nt]), ("reorder", [0, 2, 1, 3])]


def gemm_c_tiled(M: int, N: int, mt: int, nt: int):
    """C: M/mt N/nt mt nt."""
    return [("split", 0, [M // mt, mt]), ("split", 2, [N // nt, nt]), ("reorder", [0, 2, 1, 3])]


def gemm_nkn_b(K: int, N: int, n: int = 16):
    """NKn B: N/n K n (reading A12)."""
    return [("split", 1, [N // n, n]), ("reorder", [1, 0, 2])]


def transpose2():
    return [("reorder", [1, 0])]


def fold_extent(C: int, S: int):
    """(Cp, E) for the window-folded layouts: channels padded to Cp, windows
    of E >= S columns, E * Cp a power of two >= 16 (one K row of 32..128 B)."""
    Cp = 4 if C <= 4 else (C + 7) // 8 * 8
    E = 1
    while E < S or (E * Cp) < 16:
        E *= 2
    return Cp, E


def conv_input_wfold(C: int, S: int, stride: int, pad: int):
    """N H W/V E Cp: pad W by the conv padding, unfold(B = E, step = V) so
    each layout tile holds one output column's filter window (P:727-749,
    reading A23), channels innermost.  The tensor-core conv then reduces over
    the contiguous (window, channel) run — few-channel layers (conv1)."""
    Cp, E = fold_extent(C, S)
    pr = []
    if Cp > C:
        pr.append(("pad", 1, 0, Cp - C))
    # hi padding grows by E - S so the last output column's window is whole
    pr += [("pad", 3, pad, pad + E - S), ("unfold", 3, E, stride), ("reorder", [0, 2, 3, 4, 1])]
    return pr


def kcrs_wfold(K: int, C: int, S: int):
    """Weights K R E Cp for conv_input_wfold inputs (S zero-padded to E)."""
    Cp, E = fold_extent(C, S)
    pr = []
    if Cp > C:
        pr.append(("pad", 1, 0, Cp - C))
    if E > S:
        pr.append(("pad", 3, 0, E - S))
    pr.append(("reorder", [0, 2, 3, 1]))
    return pr
