"""Seeded, counter-based synthetic inputs shared by the tests, smoke() and bench.py.

This module holds NO arithmetic of the verification method: it only produces
input arrays (and the indices at which it planted mismatches).  Both the CUDA
path and the oracle receive the arrays it returns; neither imports the other.

Every element is a pure function of (seed, global index), built from integer
bit operations in torch int64 (wrapping multiply, logical shifts emulated by
masking), so the same call gives bit-identical arrays on CPU and on CUDA and
any shard [start, start+count) can be generated on its own.  Recipe
(DESIGN.md sec. 4):

  h(seed, i)  = splitmix64_finalizer(seed XOR i * 0x9E3779B97F4A7C15)
  f32 values  = ((h >> 40) - 2^23) * 2^-23              in [-1, 1)     (C1, C3)
  f32 field   = 0.5 + (h >> 41) * 2^-23                 in [0.5, 1.5)  (C2)
  f64 values  = +-(1.m) * 2^e, m = low 52 bits, e in [-16, 15]          (C3, C4)
  i32 values  = int32(h >> 32)                                          (C3, C5)
  noise       = out bits = ref bits + k, k in [-4, 4] (0 where ref == 0)
  seeds       = 2014 + config number
"""
from __future__ import annotations

import torch

MASK64 = (1 << 64) - 1


def _s64(c: int) -> int:
    c &= MASK64
    return c - (1 << 64) if c >= (1 << 63) else c


GOLDEN = _s64(0x9E3779B97F4A7C15)
MIX1 = _s64(0xBF58476D1CE4E5B9)
MIX2 = _s64(0x94D049BB133111EB)


def _srl(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of an int64 tensor holding uint64 bits."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def hash64(seed: int, idx: torch.Tensor) -> torch.Tensor:
    """h(seed, i) as int64 tensor holding the uint64 bit pattern."""
    z = idx * GOLDEN
    z = z ^ _s64(seed)
    z = (z ^ _srl(z, 30)) * MIX1
    z = (z ^ _srl(z, 27)) * MIX2
    return z ^ _srl(z, 31)


def hash64_py(seed: int, i: int) -> int:
    """Pure-Python h(seed, i) (uint64), the pin for ``hash64``."""
    z = (i * 0x9E3779B97F4A7C15) & MASK64
    z ^= seed & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def substream(seed: int, salt: int) -> int:
    """Independent seed for a named sub-stream (values, noise, injection ...)."""
    return hash64_py(seed, 0x5EED0000 + salt)


S_VALUE, S_NOISE, S_INJECT, S_SPECIAL = 1, 2, 3, 4


def _idx(start: int, count: int, device) -> torch.Tensor:
    return torch.arange(start, start + count, dtype=torch.int64, device=device)


# ----------------------------------------------------------------- value streams
def f32_uniform(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    h = hash64(substream(seed, S_VALUE), _idx(start, count, device))
    v = _srl(h, 40) - (1 << 23)
    return v.to(torch.float32) * (2.0 ** -23)


def f32_field(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    h = hash64(substream(seed, S_VALUE), _idx(start, count, device))
    return _srl(h, 41).to(torch.float32) * (2.0 ** -23) + 0.5


def f64_values(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    h = hash64(substream(seed, S_VALUE), _idx(start, count, device))
    mant = h & ((1 << 52) - 1)
    e = _srl(h, 52) & 31  # 0..31 -> exponent -16..15
    sign = _srl(h, 63)
    bits = (sign << 63) | ((e + (1023 - 16)) << 52) | mant
    return bits.view(torch.float64)


def i32_values(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    h = hash64(substream(seed, S_VALUE), _idx(start, count, device))
    return _srl(h, 32).to(torch.int32)  # wraps to the low 32 bits


def noise_k(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    h = hash64(substream(seed, S_NOISE), _idx(start, count, device))
    return (_srl(h, 1) % 9) - 4


def add_ulp_noise(ref: torch.Tensor, seed: int, start: int) -> torch.Tensor:
    """out = ref with its bit pattern moved by k in [-4, 4] ulps (k = 0 where ref == 0)."""
    k = noise_k(seed, start, ref.numel(), ref.device)
    if ref.dtype == torch.float32:
        bits = ref.view(torch.int32).to(torch.int64)
        k = torch.where(ref == 0, torch.zeros_like(k), k)
        return (bits + k).to(torch.int32).view(torch.float32)
    if ref.dtype == torch.float64:
        bits = ref.view(torch.int64)
        k = torch.where(ref == 0, torch.zeros_like(k), k)
        return (bits + k).view(torch.float64)
    raise TypeError(ref.dtype)


def distinct_indices(seed: int, count: int, lo: int, hi: int) -> list[int]:
    """First ``count`` distinct values of lo + h(seed, j) mod (hi - lo), j = 0, 1, ..."""
    out, seen, j = [], set(), 0
    span = hi - lo
    count = min(count, span)
    while len(out) < count:
        v = lo + hash64_py(seed, j) % span
        j += 1
        if v not in seen:
            seen.add(v)
            out.append(v)
    return out


# --------------------------------------------------------------- special values
F32_SPECIAL_BITS = [
    0x00000000, 0x80000000,  # +0, -0
    0x3F800000, 0xBF800000,  # +1, -1
    0x3F800001,              # 1 + ulp
    0x3F800054,              # 1.00001f
    0x3F800060,              # 1.0000115f
    0x358637BD,              # 1e-6f
    0x360637BD,              # 2e-6f = fl32(2e-6)
    0x00000001, 0x80000001,  # +-1.4e-45 (smallest subnormal)
    0x007FFFFF,              # largest subnormal
    0x7F7FFFFF, 0xFF7FFFFF,  # +-FLT_MAX
    0x7149F2CA,              # 1e30f
    0x7F61B1E6,              # 3e38f
    0x3E0DBE39, 0x3E0DBD99,  # the fp32-vs-fp64 sentinel pair
    0x7F800000, 0xFF800000,  # +-Inf
    0x7FC00000,              # qNaN
    0xFFC00001,              # negative NaN with payload
]

TOL_PAIRS = [(0.0, 0.0), (1e-6, 1e-5), (0.0, 1e-5), (1e-6, 0.0), (1.0, 1.0), (0.0, 2.0)]

from .configs import *  # noqa: E402,F401,F403
