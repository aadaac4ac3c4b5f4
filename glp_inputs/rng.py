"""Counter-based random numbers shared by every generator (splitmix64).

Both the CUDA path and the CPU oracle are fed from the same seeded inputs, and
some of those inputs are built on the GPU (RMAT-24 would take ~30 min in numpy).
A stateful RNG (torch.Generator) gives different streams on CPU and CUDA, so
every random draw here is a pure function ``hash(seed, stream, index)`` computed
with int64 torch ops that wrap identically on both devices.  The same graph is
therefore produced bit-for-bit on ``cpu`` and ``cuda`` (checked in
``tests/test_inputs.py``).

This module holds no label-propagation arithmetic.
"""
from __future__ import annotations

import torch

_M64 = (1 << 64) - 1


def _s64(x: int) -> int:
    """Reinterpret an unsigned 64-bit constant as a signed int64 literal."""
    x &= _M64
    return x - (1 << 64) if x >= (1 << 63) else x


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_MIX1 = _s64(0xBF58476D1CE4E5B9)
_MIX2 = _s64(0x94D049BB133111EB)


def _lsr(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 tensor (torch's >> is arithmetic)."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 finaliser on an int64 tensor (wrapping arithmetic)."""
    z = x + _GOLDEN
    z = (z ^ _lsr(z, 30)) * _MIX1
    z = (z ^ _lsr(z, 27)) * _MIX2
    return z ^ _lsr(z, 31)


def splitmix64_int(x: int) -> int:
    """Pure-Python splitmix64 (used to pin the tensor version in tests)."""
    z = (x + 0x9E3779B97F4A7C15) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def stream_key(seed: int, stream: int) -> int:
    """64-bit key of (seed, stream) as a signed int64 literal."""
    return _s64(splitmix64_int(((seed & 0xFFFFFFFF) << 32) ^ (stream & 0xFFFFFFFF) ^ 0x5DEECE66D))


def hash64(seed: int, stream: int, index: torch.Tensor) -> torch.Tensor:
    """Random int64 bits for every entry of ``index`` (int64 tensor)."""
    return splitmix64(index * _GOLDEN + stream_key(seed, stream))


def uniform(seed: int, stream: int, index: torch.Tensor) -> torch.Tensor:
    """float64 uniforms in [0, 1) with 53 random bits."""
    h = _lsr(hash64(seed, stream, index), 11)
    return h.to(torch.float64) * (1.0 / (1 << 53))


def uniform_pair(seed: int, stream: int, index: torch.Tensor):
    """Two float64 uniforms in [0, 1) (32 random bits each) from one hash."""
    h = hash64(seed, stream, index)
    hi = _lsr(h, 32).to(torch.float64) * (1.0 / (1 << 32))
    lo = (h & 0xFFFFFFFF).to(torch.float64) * (1.0 / (1 << 32))
    return hi, lo


def randint(seed: int, stream: int, index: torch.Tensor, high: int) -> torch.Tensor:
    """Integers in [0, high) (multiply-shift on 31 random bits; high < 2^31)."""
    assert 0 < high < (1 << 31)
    h = _lsr(hash64(seed, stream, index), 33)  # 31 bits
    return (h * high) >> 31


def permutation(seed: int, stream: int, n: int, device) -> torch.Tensor:
    """A random permutation of range(n): position of i after sorting by hash.

    Returns ``rank`` with rank[i] = new id of old id i.  Stable sort makes ties
    (probability ~n^2/2^64) resolve identically on every device.
    """
    idx = torch.arange(n, dtype=torch.int64, device=device)
    h = hash64(seed, stream, idx)
    order = torch.sort(h, stable=True).indices
    rank = torch.empty_like(order)
    rank[order] = idx
    return rank
