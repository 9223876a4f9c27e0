"""Seeded synthetic inputs.  Shared by tests, bench and the
oracle comparisons; holds none of the method's arithmetic — only random
number generation and dtype rounding."""
from __future__ import annotations

import math
import zlib

import torch


def gen(name: str) -> torch.Generator:
    return torch.Generator(device="cpu").manual_seed(zlib.crc32(name.encode()) & 0x7FFFFFFF)


def uniform(name: str, shape, lo=-1.0, hi=1.0) -> torch.Tensor:
    return torch.rand(tuple(shape), generator=gen(name), dtype=torch.float32) * (hi - lo) + lo


def activations(name: str, shape) -> torch.Tensor:
    return uniform(name, shape)


def weights(name: str, shape) -> torch.Tensor:
    fan_in = 1
    for s in shape[1:]:
        fan_in *= s
    return uniform(name, shape) / math.sqrt(fan_in)


def bn_scale(name: str, K: int) -> torch.Tensor:
    return uniform(name, (K,), 0.5, 1.5)


def bn_bias(name: str, K: int) -> torch.Tensor:
    return uniform(name, (K,), -0.1, 0.1)


def bits(name: str, shape, dtype=torch.bfloat16) -> torch.Tensor:
    """random 16/32-bit patterns (NaN payloads, -0, denormals included)"""
    g = gen(name)
    if dtype == torch.bfloat16:
        return torch.randint(-2**15, 2**15, tuple(shape), generator=g, dtype=torch.int16).view(torch.bfloat16)
    return torch.randint(-2**31, 2**31 - 1, tuple(shape), generator=g, dtype=torch.int32).view(torch.float32)
