"""ctypes binding of libalt.so (include/alt.h) — argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels; this module
only converts Python / torch arguments into the C-ABI's plain pointers and
sizes.  If the shared library is missing the import fails: there is no CPU
fallback.

Primitive sequences use plain tuples (0-based dims; paper §4.1, Table 1):
    ("split", dim, [F1, ..., Fm]), ("reorder", [p...]), ("fuse", dim, count),
    ("unfold", dim, B, S), ("pad", dim, lo, hi)
"""
from __future__ import annotations

import ctypes
import os
from typing import Iterable, Sequence

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# ALT_LIB_VARIANT=<name> loads libalt_<name>.so from this directory (developer A/B
# comparisons of kernel variants; never a CPU path)
_LIB_PATH = os.path.join(_HERE, "libalt%s.so" % ("_" + os.environ["ALT_LIB_VARIANT"] if os.environ.get("ALT_LIB_VARIANT") else ""))
if not os.path.exists(_LIB_PATH):
    raise ImportError(f"{_LIB_PATH} is missing: run __graft_entry__.build() (make -C "
                      f"{_HERE}); there is no CPU fallback")
_lib = ctypes.CDLL(_LIB_PATH)

ALT_OK, ALT_E_INVALID, ALT_E_SHAPE, ALT_E_NONDIVISIBLE = 0, 1, 2, 3
ALT_E_LOSSY, ALT_E_UNSUPPORTED, ALT_E_CUDA, ALT_E_NOMEM = 4, 5, 6, 7
ALT_F32, ALT_BF16 = 0, 1
ALT_LOSSLESS, ALT_HAS_PAD, ALT_HAS_UNFOLD, ALT_SEPARABLE, ALT_IDENTITY = 1, 2, 4, 8, 16
PATH_AUTO, PATH_TC, PATH_SIMT, PATH_DW = 0, 1, 2, 3
ACT = {None: 0, "none": 0, "relu": 1, "relu6": 2, 0: 0, 1: 1, 2: 2}
_KIND = {"split": 0, "reorder": 1, "fuse": 2, "unfold": 3, "pad": 4}
_KIND_NAME = {v: k for k, v in _KIND.items()}
MAX_RANK, MAX_PRIMS = 10, 16


class AltError(RuntimeError):
    def __init__(self, code: int, where: str):
        msg = _lib.alt_last_error().decode()
        super().__init__(f"{where}: {_lib.alt_status_str(code).decode()} ({msg})")
        self.code = code


class _Prim(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("dim", ctypes.c_int32), ("n", ctypes.c_int32),
                ("_pad", ctypes.c_int32), ("v", ctypes.c_int64 * MAX_RANK)]


class ConvParams(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in ("N", "C", "H", "W", "K", "R", "S")] + \
               [(n, ctypes.c_int32) for n in ("stride_h", "stride_w", "pad_h", "pad_w",
                                              "dil_h", "dil_w", "groups", "_pad")]


class Conv3dParams(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in ("N", "C", "D", "H", "W", "K", "T", "R", "S")] + \
               [(n, ctypes.c_int32) for n in ("stride_d", "stride_h", "stride_w", "pad_d", "pad_h", "pad_w",
                                              "dil_d", "dil_h", "dil_w", "groups")]


class _Epi(ctypes.Structure):
    _fields_ = [("scale", ctypes.c_void_p), ("bias", ctypes.c_void_p),
                ("residual", ctypes.c_void_p), ("residual_l", ctypes.c_void_p),
                ("act", ctypes.c_int32), ("flags", ctypes.c_int32)]


class KernelCfg(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("path", "block_m", "block_n", "block_k", "stages",
                                              "cta_pair", "tile_n", "tile_h", "tile_w", "split_k",
                                              "split_cluster")]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_ if n != "_pad"}


class MatmulParams(ctypes.Structure):
    _fields_ = [("M", ctypes.c_int64), ("N", ctypes.c_int64), ("K", ctypes.c_int64)]


class TuneSpace(ctypes.Structure):
    _fields_ = [("vals", (ctypes.c_int64 * 8) * 16), ("nvals", ctypes.c_int32 * 16),
                ("max_points", ctypes.c_int32), ("warmup", ctypes.c_int32),
                ("reps", ctypes.c_int32), ("fix_x", ctypes.c_int32),
                ("fixed_x", ctypes.c_void_p), ("topk", ctypes.c_int32)]


class TuneResult(ctypes.Structure):
    _fields_ = [("prims", (_Prim * MAX_PRIMS) * 3), ("nprims", ctypes.c_int32 * 3),
                ("cfg", KernelCfg), ("best_us", ctypes.c_float), ("measured", ctypes.c_int32)]


_p, _i32, _i64, _u32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32
_lib.alt_status_str.restype = ctypes.c_char_p
_lib.alt_status_str.argtypes = [ctypes.c_int]
_lib.alt_last_error.restype = ctypes.c_char_p
_lib.alt_layout_create.argtypes = [_i32, _p, _p, _i32, _p]
_lib.alt_layout_destroy.argtypes = [_p]
_lib.alt_layout_query.argtypes = [_p, _p, _p, _p, _p]
_lib.alt_layout_logical.argtypes = [_p, _p, _p]
_lib.alt_layout_phys_to_logical.argtypes = [_p, _i64, _p, _p]
_lib.alt_layout_logical_to_phys.argtypes = [_p, _p, _p]
_lib.alt_relayout.argtypes = [_p, _p, _p, _p, ctypes.c_int, _p]
_lib.alt_conv2d.argtypes = [_p, _p, _p, _p, _p, _p, _p, ctypes.c_int, _p, _p, _p]
_lib.alt_conv3d.argtypes = [_p, _p, _p, _p, _p, _p, _p, ctypes.c_int, _p, _p, _p]
_lib.alt_matmul.argtypes = [_i64, _i64, _i64, _p, _p, _p, _p, _p, _p, ctypes.c_int, _p, _p, _p]
_lib.alt_last_plan.argtypes = [_p]
_lib.alt_launch_count.restype = ctypes.c_uint64
_lib.alt_tune.argtypes = [ctypes.c_int, _p, ctypes.c_int, _p, _p, _p, _p]
_lib.alt_plan_chain.argtypes = [_i32, _p, _i32, _p, _p, _p, _p, _p, _p, _p]
_lib.alt_pool2d.argtypes = [_p, _p, _p, _p, _p, ctypes.c_int, ctypes.c_int32, _p]
_lib.alt_store_at.argtypes = [_p, _p, _p, ctypes.c_int32, _p, _p, ctypes.c_int, _p]
_lib.alt_decouple_at.argtypes = [_p, _p, ctypes.c_int32, _p, _p, _p, ctypes.c_int, _p]
_lib.alt_matmul_store_at.argtypes = [_i64, _i64, _i64, _p, _p, _p, _p, _p, _p, ctypes.c_int, _p, _p, _p]
for _f in ("alt_layout_create", "alt_layout_destroy", "alt_layout_query", "alt_layout_logical",
           "alt_layout_phys_to_logical", "alt_layout_logical_to_phys", "alt_relayout",
           "alt_conv2d", "alt_matmul", "alt_last_plan", "alt_tune", "alt_plan_chain", "alt_pool2d"):
    getattr(_lib, _f).restype = ctypes.c_int


def _check(rc: int, where: str):
    if rc != ALT_OK:
        raise AltError(rc, where)


def lib_path() -> str:
    return _LIB_PATH


def prims_to_c(prims: Sequence[tuple]):
    arr = (_Prim * max(len(prims), 1))()
    for i, p in enumerate(prims):
        k = p[0]
        arr[i].kind = _KIND[k]
        if k == "split":
            arr[i].dim, arr[i].n = p[1], len(p[2])
            for j, f in enumerate(p[2]):
                arr[i].v[j] = int(f)
        elif k == "reorder":
            arr[i].n = len(p[1])
            for j, f in enumerate(p[1]):
                arr[i].v[j] = int(f)
        elif k == "fuse":
            arr[i].dim, arr[i].n = p[1], p[2]
        elif k in ("unfold", "pad"):
            arr[i].dim = p[1]
            arr[i].v[0], arr[i].v[1] = int(p[2]), int(p[3])
        else:
            raise ValueError(f"unknown primitive {p!r}")
    return arr


def prims_from_c(arr, n: int) -> list:
    out = []
    for i in range(n):
        p = arr[i]
        k = _KIND_NAME[p.kind]
        if k == "split":
            out.append(("split", p.dim, [int(p.v[j]) for j in range(p.n)]))
        elif k == "reorder":
            out.append(("reorder", [int(p.v[j]) for j in range(p.n)]))
        elif k == "fuse":
            out.append(("fuse", p.dim, p.n))
        else:
            out.append((k, p.dim, int(p.v[0]), int(p.v[1])))
    return out


class Layout:
    """An immutable compiled layout (alt_layout_create)."""

    def __init__(self, logical_shape: Sequence[int], prims: Iterable[tuple] = ()):
        self.logical_shape = tuple(int(s) for s in logical_shape)
        self.prims = list(prims)
        shp = (ctypes.c_int64 * len(self.logical_shape))(*self.logical_shape)
        h = ctypes.c_void_p()
        _check(_lib.alt_layout_create(len(self.logical_shape), shp, prims_to_c(self.prims),
                                      len(self.prims), ctypes.byref(h)),
               f"alt_layout_create{self.logical_shape}{self.prims}")
        self._h = h
        pr = ctypes.c_int32()
        ps = (ctypes.c_int64 * MAX_RANK)()
        pn = ctypes.c_int64()
        fl = ctypes.c_uint32()
        _check(_lib.alt_layout_query(h, ctypes.byref(pr), ps, ctypes.byref(pn), ctypes.byref(fl)),
               "alt_layout_query")
        self.phys_shape = tuple(int(ps[i]) for i in range(pr.value))
        self.phys_numel = int(pn.value)
        self.flags = int(fl.value)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _lib is not None:  # (interpreter shutdown: module globals cleared)
            _lib.alt_layout_destroy(h)
            self._h = None

    @property
    def handle(self):
        return self._h

    @property
    def lossless(self):
        return bool(self.flags & ALT_LOSSLESS)

    @property
    def separable(self):
        return bool(self.flags & ALT_SEPARABLE)

    @property
    def identity(self):
        return bool(self.flags & ALT_IDENTITY)

    def phys_to_logical(self, j: int):
        out = (ctypes.c_int64 * 8)()
        valid = ctypes.c_int32()
        _check(_lib.alt_layout_phys_to_logical(self._h, int(j), out, ctypes.byref(valid)),
               "alt_layout_phys_to_logical")
        return tuple(int(out[i]) for i in range(len(self.logical_shape))) if valid.value else None

    def logical_to_phys(self, coords: Sequence[int]):
        c = (ctypes.c_int64 * len(coords))(*[int(x) for x in coords])
        j = ctypes.c_int64()
        rc = _lib.alt_layout_logical_to_phys(self._h, c, ctypes.byref(j))
        if rc == ALT_E_LOSSY:
            return None
        _check(rc, "alt_layout_logical_to_phys")
        return int(j.value)

    def empty(self, dtype=torch.bfloat16, device="cuda") -> torch.Tensor:
        return torch.empty(self.phys_shape, dtype=dtype, device=device)

    def __repr__(self):
        return f"Layout({self.logical_shape}, {self.prims}) -> {self.phys_shape}"


def _dtype_code(t: torch.Tensor) -> int:
    if t.dtype == torch.bfloat16:
        return ALT_BF16
    if t.dtype == torch.float32:
        return ALT_F32
    raise TypeError(f"unsupported dtype {t.dtype}")


def _stream_ptr(stream) -> int | None:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


def _ptr(t):
    return None if t is None else t.data_ptr()


def relayout(src_l: Layout, src: torch.Tensor, dst_l: Layout, dst: torch.Tensor, stream=None):
    """alt_relayout: dst (in dst_l) <- src (in src_l).  Bit copy."""
    _check(_lib.alt_relayout(src_l.handle, _ptr(src), dst_l.handle, _ptr(dst), _dtype_code(src),
                             _stream_ptr(stream)), "alt_relayout")
    return dst


ALT_EPI_PADS_ZERO = 1


def _epi(scale, bias, residual, residual_l, act, pads_zero=False):
    if scale is None and bias is None and residual is None and not act and not pads_zero:
        return None
    e = _Epi()
    e.scale, e.bias = _ptr(scale), _ptr(bias)
    e.residual = _ptr(residual)
    e.residual_l = residual_l.handle.value if residual_l is not None else None
    e.act = ACT[act]
    e.flags = ALT_EPI_PADS_ZERO if pads_zero else 0
    return e


def _cfg(cfg):
    if cfg is None:
        return None
    if isinstance(cfg, KernelCfg):
        return cfg
    c = KernelCfg()
    for k, v in cfg.items():
        setattr(c, k, int(v))
    return c


def conv_params(N, C, H, W, K, R, S, stride=1, pad=0, groups=1, dilation=1) -> ConvParams:
    p = ConvParams()
    p.N, p.C, p.H, p.W, p.K, p.R, p.S = N, C, H, W, K, R, S
    sh, sw = (stride, stride) if isinstance(stride, int) else stride
    ph, pw = (pad, pad) if isinstance(pad, int) else pad
    p.stride_h, p.stride_w, p.pad_h, p.pad_w = sh, sw, ph, pw
    p.dil_h, p.dil_w = (dilation, dilation) if isinstance(dilation, int) else dilation
    p.groups = groups
    return p


def conv2d(p: ConvParams, x_l: Layout, x, w_l: Layout, w, y_l: Layout, y, scale=None, bias=None,
           residual=None, residual_l: Layout | None = None, act=0, cfg=None, stream=None, pads_zero=False):
    """alt_conv2d: y (in y_l) = act(scale * conv(x, w) + bias + residual).
    pads_zero: y's pad positions already hold 0 (ALT_EPI_PADS_ZERO)."""
    e = _epi(scale, bias, residual, residual_l, act, pads_zero)
    c = _cfg(cfg)
    _check(_lib.alt_conv2d(ctypes.byref(p), x_l.handle, _ptr(x), w_l.handle, _ptr(w), y_l.handle,
                           _ptr(y), _dtype_code(x), ctypes.byref(e) if e else None,
                           ctypes.byref(c) if c else None, _stream_ptr(stream)), "alt_conv2d")
    return y


def conv3d_params(N, C, D, H, W, K, T, R, S, stride=1, pad=0, dilation=1, groups=1) -> Conv3dParams:
    """alt_conv3d_params; stride / pad / dilation: an int or a (d, h, w) triple"""
    tri = lambda v: tuple(v) if isinstance(v, (tuple, list)) else (v, v, v)  # noqa: E731
    st, pd, dl = tri(stride), tri(pad), tri(dilation)
    return Conv3dParams(N, C, D, H, W, K, T, R, S, st[0], st[1], st[2], pd[0], pd[1], pd[2], dl[0], dl[1], dl[2],
                        groups)


def conv3d(p: Conv3dParams, x_l: Layout, x, w_l: Layout, w, y_l: Layout, y, scale=None, bias=None,
           residual=None, residual_l: Layout | None = None, act=0, cfg=None, stream=None, pads_zero=False):
    """alt_conv3d (C3D): y (in y_l) = act(scale * conv3d(x, w) + bias + residual)."""
    e = _epi(scale, bias, residual, residual_l, act, pads_zero)
    c = _cfg(cfg)
    _check(_lib.alt_conv3d(ctypes.byref(p), x_l.handle, _ptr(x), w_l.handle, _ptr(w), y_l.handle,
                           _ptr(y), _dtype_code(x), ctypes.byref(e) if e else None,
                           ctypes.byref(c) if c else None, _stream_ptr(stream)), "alt_conv3d")
    return y


def matmul(M, N, K, a_l: Layout, a, b_l: Layout, b, c_l: Layout, c, scale=None, bias=None,
           residual=None, residual_l=None, act=0, cfg=None, stream=None):
    """alt_matmul: C (in c_l) = act(scale * A B + bias + residual)."""
    e = _epi(scale, bias, residual, residual_l, act)
    k = _cfg(cfg)
    _check(_lib.alt_matmul(int(M), int(N), int(K), a_l.handle, _ptr(a), b_l.handle, _ptr(b),
                           c_l.handle, _ptr(c), _dtype_code(a), ctypes.byref(e) if e else None,
                           ctypes.byref(k) if k else None, _stream_ptr(stream)), "alt_matmul")
    return c


def store_at(a_l: Layout, a, b, dim: int, z_l: Layout, z, stream=None):
    """alt_store_at: z (in z_l) = a with b attached as the last slice of dim."""
    _check(_lib.alt_store_at(a_l.handle, _ptr(a), _ptr(b), int(dim), z_l.handle, _ptr(z), _dtype_code(z),
                             _stream_ptr(stream)), "alt_store_at")
    return z


def decouple_at(z_l: Layout, z, dim: int, a_l: Layout, a, b, stream=None):
    """alt_decouple_at: the inverse of store_at; a through a_l, b dense."""
    _check(_lib.alt_decouple_at(z_l.handle, _ptr(z), int(dim), a_l.handle, _ptr(a), _ptr(b), _dtype_code(z),
                                _stream_ptr(stream)), "alt_decouple_at")
    return a, b


def matmul_store_at(M, N, K, a_l: Layout, a, z_l: Layout, z, c_l: Layout, c, scale=None, residual=None,
                    residual_l=None, act=0, cfg=None, stream=None):
    """alt_matmul_store_at: C = act(scale * A Z[:K] + Z[K] + residual), Z = store_at(B, bias, 0)."""
    e = _epi(scale, None, residual, residual_l, act)
    k = _cfg(cfg)
    _check(_lib.alt_matmul_store_at(int(M), int(N), int(K), a_l.handle, _ptr(a), z_l.handle, _ptr(z),
                                    c_l.handle, _ptr(c), _dtype_code(a), ctypes.byref(e) if e else None,
                                    ctypes.byref(k) if k else None, _stream_ptr(stream)),
           "alt_matmul_store_at")
    return c


def pool2d(p: ConvParams, x_l: Layout, x, y_l: Layout, y, kind: str = "max", stream=None):
    """alt_pool2d: max / average pooling through declared layouts."""
    _check(_lib.alt_pool2d(ctypes.byref(p), x_l.handle, _ptr(x), y_l.handle, _ptr(y), _dtype_code(x),
                           0 if kind == "max" else 1, _stream_ptr(stream)), "alt_pool2d")
    return y


def last_plan() -> dict:
    c = KernelCfg()
    _check(_lib.alt_last_plan(ctypes.byref(c)), "alt_last_plan")
    return c.as_dict()


def launch_count() -> int:
    return int(_lib.alt_launch_count())


def tune(op: str, params, dtype: int, space: dict | None = None, stream=None,
         max_points: int = 64, warmup: int = 3, reps: int = 10, fixed_x: Layout | None = None,
         topk: int = 3):
    """alt_tune over the bounded grid; returns (x/A prims, w/B prims, y/C prims, cfg, best_us,
    measured, all_us)."""
    sp = TuneSpace()
    for i, vals in (space or {}).items():
        sp.nvals[i] = len(vals)
        for j, v in enumerate(vals):
            sp.vals[i][j] = int(v)
    sp.max_points, sp.warmup, sp.reps, sp.topk = max_points, warmup, reps, topk
    if fixed_x is not None:
        sp.fix_x, sp.fixed_x = 1, fixed_x.handle.value
    res = TuneResult()
    all_us = (ctypes.c_float * max(max_points, 1))()
    kind = 0 if op == "conv2d" else 1
    _check(_lib.alt_tune(kind, ctypes.byref(params), dtype, ctypes.byref(sp), _stream_ptr(stream),
                         ctypes.byref(res), all_us), "alt_tune")
    seqs = [prims_from_c(res.prims[i], res.nprims[i]) for i in range(3)]
    return dict(x=seqs[0], w=seqs[1], y=seqs[2], cfg=res.cfg.as_dict(), best_us=res.best_us,
                measured=res.measured, all_us=[all_us[i] for i in range(res.measured)])


def plan_chain(op_kind: Sequence[int], edges: Sequence[tuple], edge_layouts: Sequence[Layout | None]):
    """alt_plan_chain (Alg. 1).  edges = [(src_op, dst_op, in_idx, numel)], -1 = none.
    Returns (src_edge list, conversion list)."""
    n_ops, n_e = len(op_kind), len(edges)
    ok = (ctypes.c_int32 * max(n_ops, 1))(*op_kind)
    es = (ctypes.c_int32 * max(n_e, 1))(*[e[0] for e in edges])
    ed = (ctypes.c_int32 * max(n_e, 1))(*[e[1] for e in edges])
    ei = (ctypes.c_int32 * max(n_e, 1))(*[e[2] for e in edges])
    en = (ctypes.c_int64 * max(n_e, 1))(*[e[3] for e in edges])
    el = (ctypes.c_void_p * max(n_e, 1))(*[(l.handle.value if l is not None else None)
                                           for l in edge_layouts])
    se = (ctypes.c_int32 * max(n_e, 1))()
    cv = (ctypes.c_int32 * max(n_e, 1))()
    _check(_lib.alt_plan_chain(n_ops, ok, n_e, es, ed, ei, en, el, se, cv), "alt_plan_chain")
    return [se[i] for i in range(n_e)], [cv[i] for i in range(n_e)]


EXPORTED = ["alt_status_str", "alt_last_error", "alt_layout_create", "alt_layout_destroy",
            "alt_layout_query", "alt_layout_logical", "alt_layout_phys_to_logical",
            "alt_layout_logical_to_phys", "alt_relayout", "alt_conv2d", "alt_matmul",
            "alt_last_plan", "alt_launch_count", "alt_tune", "alt_plan_chain", "alt_pool2d",
            "alt_store_at", "alt_decouple_at", "alt_matmul_store_at", "alt_conv3d"]
