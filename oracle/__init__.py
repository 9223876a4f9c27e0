"""fp64 CPU oracle for ALT's hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` leg / ``--impl reference`` arm may import this package.  It
shares no code with the product package (``paper_conf_eurosys_xuxpwwwdxcwc23_b200``)
or ``include/``; the C side (``alt_oracle.c``) re-derives every map from the
paper.  See the header of ``alt_oracle.c`` for the O1-O6 definitions and their
PAPER.md citations; ``oracle/propagate.py`` holds O7 (Algorithm 1).

Primitive sequences are plain tuples (0-based dims, reading A1):
    ("split", dim, [F1, ..., Fm])     Table 1
    ("reorder", [p0, ..., pr-1])      Table 1
    ("fuse", dim, count)              Table 1
    ("unfold", dim, B, S)             §4.1.2
    ("pad", dim, lo, hi)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "alt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

E_OK, E_INVALID, E_SHAPE, E_NONDIV, E_LOSSY = 0, 1, 2, 3, 4
_KINDS = {"split": 0, "reorder": 1, "fuse": 2, "unfold": 3, "pad": 4}


class OracleError(Exception):
    def __init__(self, code: int, what: str = ""):
        super().__init__(f"oracle error {code} {what}")
        self.code = code


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (-O2, OpenMP, fp64)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-o", _LIB, _SRC, "-lm"]
        )
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        c_ll, c_p, c_i = ctypes.c_longlong, ctypes.c_void_p, ctypes.c_int
        L.orc_layout_sizeof.restype = c_ll
        L.orc_layout_build.restype = c_i
        L.orc_layout_build.argtypes = [c_i, c_p, c_i, c_p, c_p, c_p, c_p, c_p]
        L.orc_phys_rank.argtypes = [c_p]
        L.orc_phys_rank.restype = c_i
        L.orc_phys_shape.argtypes = [c_p, c_p]
        L.orc_phys_numel.argtypes = [c_p]
        L.orc_phys_numel.restype = c_ll
        L.orc_G.argtypes = [c_p, c_p, c_p]
        L.orc_G.restype = c_i
        L.orc_F.argtypes = [c_p, c_p, c_p]
        L.orc_F.restype = c_i
        L.orc_G_linear.argtypes = [c_p, c_ll, c_p]
        L.orc_G_linear.restype = c_i
        L.orc_F_linear.argtypes = [c_p, c_p]
        L.orc_F_linear.restype = c_ll
        for f in ("orc_materialize", "orc_unmaterialize"):
            getattr(L, f).argtypes = [c_p, c_p, c_p, c_i]
            getattr(L, f).restype = c_i
        L.orc_check_consistent.argtypes = [c_p, c_p, c_i]
        L.orc_check_consistent.restype = c_ll
        L.orc_relayout.argtypes = [c_p, c_p, c_p, c_p, c_i]
        L.orc_relayout.restype = c_i
        L.orc_read_logical.argtypes = [c_p, c_p, c_i, c_p]
        L.orc_read_logical.restype = c_i
        L.orc_present_mask.argtypes = [c_p, c_p]
        L.orc_conv2d_f64.argtypes = [c_p, c_p, c_p, c_p, c_p, c_p, c_i, c_ll, c_ll, c_p]
        L.orc_conv3d_f64.argtypes = [c_p, c_p, c_p, c_p, c_p, c_p, c_i, c_p]
        L.orc_conv2d_points.argtypes = [c_p, c_p, c_p, c_p, c_p, c_i, c_p, c_p, c_p, c_p,
                                        c_i, c_ll, c_p, c_p]
        L.orc_conv2d_points.restype = c_i
        L.orc_conv2d_unfold_native.argtypes = [c_p, c_ll, c_ll, c_p, c_p, c_p]
        L.orc_gemm_f64.argtypes = [c_ll, c_ll, c_ll, c_p, c_p, c_p, c_p, c_p, c_i,
                                   c_ll, c_ll, c_p]
        L.orc_pool2d_f64.argtypes = [c_p, c_p, c_i, c_p]
        _lib = L
    return _lib


def _ptr(a: np.ndarray | None):
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.c_void_p)


def _wb(arr: np.ndarray) -> int:
    if arr.dtype.itemsize not in (2, 4):
        raise ValueError("words must be 16- or 32-bit")
    return arr.dtype.itemsize


class Layout:
    """O1: a logical row-major tensor transformed by a primitive sequence."""

    def __init__(self, logical_shape: Sequence[int], prims: Sequence[tuple] = ()):
        L = lib()
        self.logical_shape = tuple(int(s) for s in logical_shape)
        self.prims = list(prims)
        npr = len(self.prims)
        kinds = np.zeros(max(npr, 1), np.int32)
        dims = np.zeros(max(npr, 1), np.int32)
        ns = np.zeros(max(npr, 1), np.int32)
        vals = np.zeros((max(npr, 1), 10), np.int64)
        for i, p in enumerate(self.prims):
            kind = p[0]
            kinds[i] = _KINDS[kind]
            if kind == "split":
                dims[i], ns[i] = p[1], len(p[2])
                vals[i, : len(p[2])] = p[2]
            elif kind == "reorder":
                ns[i] = len(p[1])
                vals[i, : len(p[1])] = p[1]
            elif kind == "fuse":
                dims[i], ns[i] = p[1], p[2]
            elif kind == "unfold":
                dims[i] = p[1]
                vals[i, 0], vals[i, 1] = p[2], p[3]
            elif kind == "pad":
                dims[i] = p[1]
                vals[i, 0], vals[i, 1] = p[2], p[3]
        self._buf = ctypes.create_string_buffer(int(L.orc_layout_sizeof()))
        ls = np.array(self.logical_shape, np.int64)
        rc = L.orc_layout_build(len(ls), _ptr(ls), npr, _ptr(kinds), _ptr(dims), _ptr(ns),
                                _ptr(vals), self._buf)
        if rc != E_OK:
            raise OracleError(rc, f"layout {self.logical_shape} {self.prims}")
        pr = L.orc_phys_rank(self._buf)
        ps = np.zeros(12, np.int64)
        L.orc_phys_shape(self._buf, _ptr(ps))
        self.phys_shape = tuple(int(x) for x in ps[:pr])
        self.phys_numel = int(np.prod(self.phys_shape))
        self.logical_numel = int(np.prod(self.logical_shape))

    @property
    def handle(self):
        return self._buf

    def G(self, phys: Sequence[int]):
        """physical coords -> logical coords, or None for a structural zero."""
        c = np.array(phys, np.int64)
        out = np.zeros(12, np.int64)
        ok = lib().orc_G(self._buf, _ptr(c), _ptr(out))
        return tuple(int(x) for x in out[: len(self.logical_shape)]) if ok else None

    def F(self, logical: Sequence[int]):
        """logical coords -> owner physical coords, or None if no copy."""
        c = np.array(logical, np.int64)
        out = np.zeros(12, np.int64)
        ok = lib().orc_F(self._buf, _ptr(c), _ptr(out))
        return tuple(int(x) for x in out[: len(self.phys_shape)]) if ok else None

    def G_linear(self, j: int):
        out = np.zeros(12, np.int64)
        ok = lib().orc_G_linear(self._buf, int(j), _ptr(out))
        return tuple(int(x) for x in out[: len(self.logical_shape)]) if ok else None

    def F_linear(self, logical: Sequence[int]) -> int:
        c = np.array(logical, np.int64)
        return int(lib().orc_F_linear(self._buf, _ptr(c)))

    # ---------------------------------------------------------------- O2 --
    def materialize(self, logical: np.ndarray) -> np.ndarray:
        logical = np.ascontiguousarray(logical)
        assert logical.shape == self.logical_shape, (logical.shape, self.logical_shape)
        out = np.empty(self.phys_shape, logical.dtype)
        rc = lib().orc_materialize(self._buf, _ptr(logical), _ptr(out), _wb(logical))
        if rc != E_OK:
            raise OracleError(rc)
        return out

    def unmaterialize(self, phys: np.ndarray) -> np.ndarray:
        phys = np.ascontiguousarray(phys).reshape(self.phys_shape)
        out = np.empty(self.logical_shape, phys.dtype)
        rc = lib().orc_unmaterialize(self._buf, _ptr(phys), _ptr(out), _wb(phys))
        if rc != E_OK:
            raise OracleError(rc, "lossy")
        return out

    def check_consistent(self, phys: np.ndarray) -> int:
        phys = np.ascontiguousarray(phys).reshape(self.phys_shape)
        return int(lib().orc_check_consistent(self._buf, _ptr(phys), _wb(phys)))

    def read_f64(self, phys: np.ndarray, allow_lossy: bool = False) -> np.ndarray:
        """Logical fp64 values of a physical buffer of fp32 (uint32 / float32)
        or bf16 (uint16) words.  A lossy layout raises unless allow_lossy, in
        which case elements without a copy read as 0 (see present())."""
        phys = np.ascontiguousarray(phys).reshape(self.phys_shape)
        if phys.dtype == np.float32:
            phys = phys.view(np.uint32)
        out = np.empty(self.logical_shape, np.float64)
        rc = lib().orc_read_logical(self._buf, _ptr(phys), _wb(phys), _ptr(out))
        if rc != E_OK and not allow_lossy:
            raise OracleError(rc, "lossy")
        return out

    def present(self) -> np.ndarray:
        """bool mask over the logical tensor: elements that have a copy."""
        m = np.empty(self.logical_shape, np.uint8)
        lib().orc_present_mask(self._buf, _ptr(m))
        return m.astype(bool)


def relayout(src_l: Layout, src: np.ndarray, dst_l: Layout) -> np.ndarray:
    """O2 conversion operator (Fig. 5a): dst = src read through src_l, stored
    through dst_l."""
    src = np.ascontiguousarray(src).reshape(src_l.phys_shape)
    out = np.empty(dst_l.phys_shape, src.dtype)
    rc = lib().orc_relayout(src_l.handle, _ptr(src), dst_l.handle, _ptr(out), _wb(src))
    if rc != E_OK:
        raise OracleError(rc, "relayout")
    return out


def _f64(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.float64)


def conv2d_f64(p: dict, x: np.ndarray, w: np.ndarray, scale=None, bias=None,
               residual=None, act: int = 0, images: tuple | None = None) -> np.ndarray:
    """O3 + O6 on fp64 logical arrays x[N,C,H,W], w[K,C/g,R,S]."""
    N, C, H, W, K, R, S = (p[k] for k in "NCHWKRS")
    Vh, Vw = p.get("stride_h", 1), p.get("stride_w", 1)
    ph, pw = p.get("pad_h", 0), p.get("pad_w", 0)
    g = p.get("groups", 1)
    dh, dw = p.get("dil_h", 1), p.get("dil_w", 1)
    Ho, Wo = (H + 2 * ph - dh * (R - 1) - 1) // Vh + 1, (W + 2 * pw - dw * (S - 1) - 1) // Vw + 1
    pr = np.array([N, C, H, W, K, R, S, Vh, Vw, ph, pw, g, dh, dw], np.int64)
    x, w = _f64(x), _f64(w)
    assert x.shape == (N, C, H, W) and w.shape == (K, C // g, R, S)
    y = np.zeros((N, K, Ho, Wo), np.float64)
    n0, n1 = images if images is not None else (0, N)
    res = _f64(residual)
    lib().orc_conv2d_f64(_ptr(pr), _ptr(x), _ptr(w), _ptr(_f64(scale)), _ptr(_f64(bias)),
                         _ptr(res), int(act), int(n0), int(n1), _ptr(y))
    return y


def conv2d(p: dict, x_l: Layout, x: np.ndarray, w_l: Layout, w: np.ndarray,
           scale=None, bias=None, res_l: Layout | None = None, residual=None,
           act: int = 0, images: tuple | None = None) -> np.ndarray:
    """O3 + O6 with operands given as physical word buffers in declared
    layouts (read exactly through each layout's F map).  The input may be a
    lossy template (reading A32: e.g. a stride-2 window narrower than its
    stride skips pixels): the conv's sum reads only pixels h = p V - pad +
    r d, w = q V - pad + s d (Eq. (1)), so x may omit others — if a pixel the
    sum reads has no copy, this refuses (OracleError)."""
    xl = x_l.read_f64(x, allow_lossy=True)
    present = x_l.present()
    if not present.all():
        g = lambda k, d=0: p.get(k, d)  # noqa: E731
        V = (g("stride_h", 1), g("stride_w", 1)); pad = (g("pad_h"), g("pad_w")); dl = (g("dil_h", 1), g("dil_w", 1))
        ext = (p["H"], p["W"])
        win = (p["R"], p["S"])
        need = []
        for a in range(2):
            out = (ext[a] + 2 * pad[a] - dl[a] * (win[a] - 1) - 1) // V[a] + 1
            idx = {o * V[a] - pad[a] + t * dl[a] for o in range(out) for t in range(win[a])}
            need.append(sorted(i for i in idx if 0 <= i < ext[a]))
        if not present[:, :, need[0]][:, :, :, need[1]].all():
            raise OracleError(E_LOSSY, "the conv reads a pixel the input layout does not hold")
    wl = w_l.read_f64(w)
    rl = res_l.read_f64(residual) if residual is not None else None
    return conv2d_f64(p, xl, wl, scale, bias, rl, act, images)


def conv3d_out(p: dict):
    """(Do, Ho, Wo) of a 3-D conv (the standard definition, as O3)."""
    g = lambda k, d=1: p.get(k, d)  # noqa: E731
    D, H, W, T, R, S = (p[k] for k in "DHWTRS")
    return ((D + 2 * g("pad_d", 0) - g("dil_d") * (T - 1) - 1) // g("stride_d") + 1,
            (H + 2 * g("pad_h", 0) - g("dil_h") * (R - 1) - 1) // g("stride_h") + 1,
            (W + 2 * g("pad_w", 0) - g("dil_w") * (S - 1) - 1) // g("stride_w") + 1)


def conv3d_f64(p: dict, x: np.ndarray, w: np.ndarray, scale=None, bias=None,
               residual=None, act: int = 0) -> np.ndarray:
    """O3b (C3D) + O6 on fp64 logical arrays x[N,C,D,H,W],
    w[K,C/g,T,R,S] -> y[N,K,Do,Ho,Wo]."""
    N, C, D, H, W, K, T, R, S = (p[k] for k in ("N", "C", "D", "H", "W", "K", "T", "R", "S"))
    g = lambda k, d=1: p.get(k, d)  # noqa: E731
    pr = np.array([N, C, D, H, W, K, T, R, S, g("stride_d"), g("stride_h"), g("stride_w"), g("pad_d", 0),
                   g("pad_h", 0), g("pad_w", 0), g("dil_d"), g("dil_h"), g("dil_w"), g("groups")], np.int64)
    x, w = _f64(x), _f64(w)
    assert x.shape == (N, C, D, H, W) and w.shape == (K, C // g("groups"), T, R, S)
    y = np.zeros((N, K) + conv3d_out(p), np.float64)
    lib().orc_conv3d_f64(_ptr(pr), _ptr(x), _ptr(w), _ptr(_f64(scale)), _ptr(_f64(bias)), _ptr(_f64(residual)),
                         int(act), _ptr(y))
    return y


def conv3d(p: dict, x_l: Layout, x: np.ndarray, w_l: Layout, w: np.ndarray, scale=None, bias=None,
           res_l: Layout | None = None, residual=None, act: int = 0) -> np.ndarray:
    """O3b + O6 with operands as physical word buffers in declared layouts."""
    return conv3d_f64(p, x_l.read_f64(x), w_l.read_f64(w), scale, bias,
                      res_l.read_f64(residual) if residual is not None else None, act)


def conv2d_points(p: dict, x_l: Layout, x: np.ndarray, w_l: Layout, w: np.ndarray,
                  pts: np.ndarray, scale=None, bias=None, res_l=None, residual=None,
                  act: int = 0) -> np.ndarray:
    """O3 + O6 evaluated at chosen outputs (n,k,p,q), reading through F."""
    N, C, H, W, K, R, S = (p[k] for k in "NCHWKRS")
    pr = np.array([N, C, H, W, K, R, S, p.get("stride_h", 1), p.get("stride_w", 1),
                   p.get("pad_h", 0), p.get("pad_w", 0), p.get("groups", 1), p.get("dil_h", 1),
                   p.get("dil_w", 1)], np.int64)
    x = np.ascontiguousarray(x)
    w = np.ascontiguousarray(w)
    if x.dtype == np.float32:
        x, w = x.view(np.uint32), w.view(np.uint32)
    if residual is not None:
        residual = np.ascontiguousarray(residual)
        if residual.dtype == np.float32:
            residual = residual.view(np.uint32)
    pts = np.ascontiguousarray(pts, dtype=np.int64)
    out = np.zeros(len(pts), np.float64)
    rc = lib().orc_conv2d_points(_ptr(pr), x_l.handle, _ptr(x), w_l.handle, _ptr(w), _wb(x),
                                 _ptr(_f64(scale)), _ptr(_f64(bias)),
                                 res_l.handle if res_l is not None else None,
                                 _ptr(residual), int(act), len(pts), _ptr(pts), _ptr(out))
    if rc != E_OK:
        raise OracleError(rc, "points")
    return out


def conv2d_unfold_native(p: dict, ht: int, wt: int, xu: np.ndarray, w: np.ndarray) -> np.ndarray:
    """O4: Fig. 3 loop nest on the Fig. 2 overlapped-tiled input through Eq. (1)."""
    N, C, H, W, K, R, S = (p[k] for k in "NCHWKRS")
    Vh, Vw = p.get("stride_h", 1), p.get("stride_w", 1)
    ph, pw = p.get("pad_h", 0), p.get("pad_w", 0)
    Ho, Wo = (H + 2 * ph - R) // Vh + 1, (W + 2 * pw - S) // Vw + 1
    pr = np.array([N, C, H, W, K, R, S, Vh, Vw, ph, pw, 1], np.int64)
    y = np.zeros((N, K, Ho, Wo), np.float64)
    lib().orc_conv2d_unfold_native(_ptr(pr), int(ht), int(wt), _ptr(_f64(xu)), _ptr(_f64(w)),
                                   _ptr(y))
    return y


def gemm_f64(A: np.ndarray, B: np.ndarray, scale=None, bias=None, residual=None,
             act: int = 0, rows: tuple | None = None) -> np.ndarray:
    """O5 + O6: C = A B in fp64, k ascending."""
    A, B = _f64(A), _f64(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    C = np.zeros((M, N), np.float64)
    m0, m1 = rows if rows is not None else (0, M)
    lib().orc_gemm_f64(M, N, K, _ptr(A), _ptr(B), _ptr(_f64(scale)), _ptr(_f64(bias)),
                       _ptr(_f64(residual)), int(act), int(m0), int(m1), _ptr(C))
    return C


def gemm(a_l: Layout, a, b_l: Layout, b, scale=None, bias=None, res_l=None, residual=None,
         act: int = 0, rows: tuple | None = None) -> np.ndarray:
    A = a_l.read_f64(a)
    B = b_l.read_f64(b)
    R = res_l.read_f64(residual) if residual is not None else None
    return gemm_f64(A, B, scale, bias, R, act, rows)


def pool2d_f64(x: np.ndarray, R: int, S: int, stride: int, pad: int, kind: str = "max") -> np.ndarray:
    """O9: max / average pooling over in-bounds taps (support op)."""
    x = _f64(x)
    N, C, H, W = x.shape
    Ho, Wo = (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1
    pr = np.array([N, C, H, W, R, S, stride, stride, pad, pad], np.int64)
    y = np.zeros((N, C, Ho, Wo), np.float64)
    lib().orc_pool2d_f64(_ptr(pr), _ptr(x), 0 if kind == "max" else 1, _ptr(y))
    return y


def bf16_bits_to_f64(u16: np.ndarray) -> np.ndarray:
    return (u16.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
