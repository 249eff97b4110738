"""Seeded synthetic input generators shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic: it only produces inputs.
Both the tests (oracle side) and the product benchmarks import it; nothing
else is shared between ``oracle/`` and the CUDA path.

Counter-based splitmix64: element i of a stream with seed
s is ``mix(s + (i+1) * 0x9E3779B97F4A7C15)`` where ``mix`` is the splitmix64
finaliser.  Because it is counter-based, shard r of a G-way split generates
exactly the same values as the corresponding slice of the unsharded stream
(``start`` argument), on CPU or on CUDA: all arithmetic is torch int64 with
two's-complement wrap, logical right shifts are emulated with masks.

Workload recipes:

sort keys (32-bit; returned as torch.int32 holding the bit pattern)
  uniform   key = z >> 32                      (full 32-bit range)
  paper     key = (z >> 1) mod 2n              (uniform in [0, 2n-1])
  sorted    key = i * floor(2^32 / n)
  reverse   key = (n-1-i) * floor(2^32 / n)
  few       key = (z >> 32) & 15               (16 distinct keys: heavy ties)
  equal     key = 7
  For key_type "f32" the 32-bit integer k is mapped to float32(int32(k)) * 2^-20,
  and every element with (z & 31) == 0 is replaced by +0.0 or -0.0 (bit 5 of z)
  so that the stable ordering of +/-0 is exercised.  No NaN, no inf.
values     val = i (global index), so stability is observable.
max-subarray (int32)
  uniform   x = int32(z >> 32)                 (full range)
  small     x = ((z >> 32) mod 2001) - 1000
  negative  x = -1 - ((z >> 32) mod 1000000)
  positive  x =  1 + ((z >> 32) mod 1000000)
  zero      x = 0
"""
from __future__ import annotations

import torch

GOLDEN = 0x9E3779B97F4A7C15
C1 = 0xBF58476D1CE4E5B9
C2 = 0x94D049BB133111EB

SORT_DISTS = ("uniform", "paper", "sorted", "reverse", "few", "equal")
MAXSUB_DISTS = ("uniform", "small", "negative", "positive", "zero")


def _s64(c: int) -> int:
    """Reinterpret a 64-bit unsigned constant as signed int64."""
    return c - (1 << 64) if c >= (1 << 63) else c


def _srl(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def splitmix64(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    """z_i for global indices i in [start, start+count), as int64 bit patterns."""
    i = torch.arange(start + 1, start + count + 1, dtype=torch.int64, device=device)
    z = i * _s64(GOLDEN) + _s64(seed & ((1 << 64) - 1))
    z = (z ^ _srl(z, 30)) * _s64(C1)
    z = (z ^ _srl(z, 27)) * _s64(C2)
    return z ^ _srl(z, 31)


def splitmix64_py(seed: int, i: int) -> int:
    """Pure-Python reference of one element (used to pin the torch version)."""
    m = (1 << 64) - 1
    z = (seed + (i + 1) * GOLDEN) & m
    z = ((z ^ (z >> 30)) * C1) & m
    z = ((z ^ (z >> 27)) * C2) & m
    return z ^ (z >> 31)


def _to_i32_bits(v: torch.Tensor) -> torch.Tensor:
    """int64 values in [0, 2^32) -> int32 tensor with the same low 32 bits."""
    v = v & 0xFFFFFFFF
    return torch.where(v >= (1 << 31), v - (1 << 32), v).to(torch.int32)


def sort_keys(n: int, dist: str = "uniform", seed: int = 1, key_type: str = "u32",
              start: int = 0, count: int | None = None, device="cpu") -> torch.Tensor:
    """Keys for global indices [start, start+count) of an n-element workload.

    Returns torch.int32 (u32/i32: the 32-bit pattern) or torch.float32 (f32).
    """
    if count is None:
        count = n - start
    if dist not in SORT_DISTS:
        raise ValueError(f"unknown sort distribution {dist!r}")
    z = splitmix64(seed, start, count, device)
    i = torch.arange(start, start + count, dtype=torch.int64, device=device)
    if dist == "uniform":
        k = _srl(z, 32)
    elif dist == "paper":
        # top 63 bits of z, so the modulus is taken on a non-negative int64
        k = _srl(z, 1) % (2 * n)
    elif dist == "sorted":
        k = i * ((1 << 32) // max(n, 1))
    elif dist == "reverse":
        k = (n - 1 - i) * ((1 << 32) // max(n, 1))
    elif dist == "few":
        k = _srl(z, 32) & 15
    else:  # equal
        k = torch.full_like(i, 7)
    bits = _to_i32_bits(k)
    if key_type in ("u32", "i32"):
        return bits
    if key_type != "f32":
        raise ValueError(f"unknown key type {key_type!r}")
    f = bits.to(torch.float32) * (2.0 ** -20)
    zero_mask = (z & 31) == 0
    neg = ((z >> 5) & 1) == 1
    zeros = torch.where(neg, torch.full_like(f, -0.0), torch.zeros_like(f))
    return torch.where(zero_mask, zeros, f)


def sort_vals(n: int, start: int = 0, count: int | None = None, device="cpu") -> torch.Tensor:
    """val[i] = i (global index) as torch.int32 bit pattern of a uint32."""
    if count is None:
        count = n - start
    return _to_i32_bits(torch.arange(start, start + count, dtype=torch.int64, device=device))


def maxsub_input(n: int, dist: str = "uniform", seed: int = 2, start: int = 0,
                 count: int | None = None, device="cpu") -> torch.Tensor:
    """int32 values for the max-subarray instance."""
    if count is None:
        count = n - start
    if dist not in MAXSUB_DISTS:
        raise ValueError(f"unknown max-subarray distribution {dist!r}")
    z = splitmix64(seed, start, count, device)
    hi = _srl(z, 32)
    if dist == "uniform":
        return _to_i32_bits(hi)
    if dist == "small":
        return ((hi % 2001) - 1000).to(torch.int32)
    if dist == "negative":
        return (-1 - (hi % 1000000)).to(torch.int32)
    if dist == "positive":
        return (1 + (hi % 1000000)).to(torch.int32)
    return torch.zeros(count, dtype=torch.int32, device=device)
