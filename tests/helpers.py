"""Shared test helpers: GPU <-> oracle marshalling and the parity bars.

Parity bars (BASELINE.json north_star; readings A13/A14 in DESIGN.md):
  relayout            bit-exact (compared as integer words)
  fp32 conv / GEMM    max|y - ref| / max|ref| <= 1e-5
  bf16 conv / GEMM    ||y - ref||_2 / ||ref||_2 <= 2e-2
The reference is the fp64 oracle evaluated on the exact operand values the
GPU read (bf16 inputs are the RNE-rounded values, converted exactly).
"""
from __future__ import annotations

import numpy as np
import torch

import oracle
from paper_conf_eurosys_xuxpwwwdxcwc23_b200 import synth

FP32_TOL = 1e-5
BF16_TOL = 2e-2


def words(t: torch.Tensor) -> np.ndarray:
    """Raw 16/32-bit words of a tensor (any device) as numpy."""
    t = t.detach().contiguous().cpu()
    if t.dtype in (torch.bfloat16, torch.float16, torch.int16):
        return t.view(torch.int16).numpy().view(np.uint16)
    return t.view(torch.int32).numpy().view(np.uint32)


def from_words(w: np.ndarray, dtype, device="cuda") -> torch.Tensor:
    if dtype == torch.bfloat16:
        return torch.from_numpy(w.view(np.int16).copy()).view(torch.bfloat16).to(device)
    return torch.from_numpy(w.view(np.int32).copy()).view(torch.float32).to(device)


def maxnorm_rel(got: np.ndarray, ref: np.ndarray) -> float:
    den = np.max(np.abs(ref))
    return float(np.max(np.abs(got - ref)) / (den if den > 0 else 1.0))


def norm_rel(got: np.ndarray, ref: np.ndarray) -> float:
    den = np.linalg.norm(ref.ravel())
    return float(np.linalg.norm((got - ref).ravel()) / (den if den > 0 else 1.0))


def assert_parity(got: np.ndarray, ref: np.ndarray, dtype):
    if dtype == torch.float32:
        err = maxnorm_rel(got, ref)
        assert err <= FP32_TOL, f"fp32 max-norm relative error {err:.3e} > {FP32_TOL}"
    else:
        err = norm_rel(got, ref)
        assert err <= BF16_TOL, f"bf16 normwise relative error {err:.3e} > {BF16_TOL}"
    return err


def make_operand(name: str, layout_prims, logical: torch.Tensor, dtype, device="cuda"):
    """Materialise a logical fp32 tensor (rounded to dtype) into a layout with
    the ORACLE (O2), upload it; returns (oracle layout, words, device tensor)."""
    lw = words(logical.to(dtype))
    OL = oracle.Layout(tuple(logical.shape), layout_prims)
    phys = OL.materialize(lw)
    return OL, phys, from_words(phys, dtype, device)


def read_output(OL: oracle.Layout, y: torch.Tensor, dtype) -> np.ndarray:
    """GPU output (physical) -> logical fp64 through the oracle's F, after
    checking every pad position is 0 and every unfold copy is equal."""
    w = words(y).reshape(OL.phys_shape)
    bad = OL.check_consistent(w)
    assert bad == 0, f"{bad} inconsistent physical positions (pad != 0 or copies differ)"
    return OL.read_f64(w)


# Per-element bar next to the normwise one (bf16 path): the GPU's error on
# every output is bounded by its bf16 output rounding (unit roundoff 2^-8 of
# |y|) plus the fp32 accumulation error (<= n 2^-24 sum |x w| |scale|, n <=
# 4608 reduction terms < 2^-11).  2^-7 (|ref| + absref) is a safe envelope
# of both; a corrupted or misplaced element (a wrong row, a stale tile)
# exceeds it.  absref = |scale| conv(|x|, |w|) + |bias| + |residual| in fp64.
ELEM_REL = 2.0 ** -7


def assert_elementwise(got: np.ndarray, ref: np.ndarray, absref: np.ndarray, what=""):
    bad = np.abs(got - ref) > ELEM_REL * (np.abs(ref) + absref)
    n = int(bad.sum())
    if n:
        idx = np.argwhere(bad)[0]
        raise AssertionError(f"{what}: {n} element(s) outside 2^-7 (|ref| + sum|x w|), first at {tuple(idx)}: "
                             f"got {got[tuple(idx)]!r} ref {ref[tuple(idx)]!r} absref {absref[tuple(idx)]!r}")


def abs_conv_ref(p: dict, xl: np.ndarray, wl: np.ndarray, scale=None, bias=None, res=None) -> np.ndarray:
    """|scale| conv(|x|, |w|) + |bias| + |res| (fp64 oracle, logical operands)"""
    return oracle.conv2d_f64(p, np.abs(xl), np.abs(wl), None if scale is None else np.abs(scale),
                             None if bias is None else np.abs(bias), None if res is None else np.abs(res), 0)
