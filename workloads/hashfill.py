"""Hash-filled inputs and their closed-form check ("at scale").

A buffer packed under layout L is filled with src[h] = H(x(h)), where x(h) is the
logical flat index that hardware index h holds and H(x) is the low w bytes of
splitmix64(x ^ seed).  Such a buffer is A-consistent by construction (equal logical
index -> equal bytes, §8(b)), for any layout including broadcasting ones, and the
conversion to B is then known in closed form at every element:
    dst[h] = H(B(h))        (O5: convert(pack_A(T)) == pack_B(T) with T = H).
So a 2^30-element conversion is checked element by element without materialising the
oracle's tables.

This module is an input generator shared by the tests and bench.py: it evaluates
x(h) from a layout's literal spec (workloads/configs.py format: the logical bit each
input bit carries) with plain torch integer ops, chunk by chunk, on whatever device
the caller passes.  It holds none of the planner's or kernels' arithmetic, and the
CPU tests pin it against the oracle's O2 apply and a scalar splitmix64
(tests/test_hashfill.py).
"""
from __future__ import annotations

from typing import List, Optional

from . import configs as W

_MASK64 = (1 << 64) - 1


def _s64(c: int) -> int:
    c &= _MASK64
    return c - (1 << 64) if c >= (1 << 63) else c


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_M1 = _s64(0xBF58476D1CE4E5B9)
_M2 = _s64(0x94D049BB133111EB)


def splitmix64_scalar(x: int) -> int:
    """Reference splitmix64 finaliser on Python ints (Steele, Lea, Flood 2014)."""
    z = (x + 0x9E3779B97F4A7C15) & _MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _MASK64
    return z ^ (z >> 31)


def _srl(x, s: int):
    """Logical right shift of an int64 tensor (torch's >> is arithmetic)."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def splitmix64(x):
    """splitmix64 of an int64 torch tensor (two's-complement wrap-around arithmetic)."""
    z = x + _GOLDEN
    z = (z ^ _srl(z, 30)) * _M1
    z = (z ^ _srl(z, 27)) * _M2
    return z ^ _srl(z, 31)


def spec_cols(spec) -> List[int]:
    """Logical flat index of every input bit of a literal layout spec (0 = broadcast),
    in the packed order of §8(b): input dims in declaration order, bit 0 first."""
    in_dims, out_dims, bases = W.spec_to_bases(spec)
    cols = []
    for name, nb in in_dims:
        for coords in bases[name]:
            x = 0
            for (dn, db), c in zip(out_dims, coords):
                x = (x << db) | int(c)
            cols.append(x)
    return cols


def logical_index(cols: List[int], h):
    """x(h) = XOR over the set bits k of h of cols[k] (int64 tensor h)."""
    x = h.new_zeros(h.shape)
    for k, c in enumerate(cols):
        if c:
            x ^= ((h >> k) & 1) * c
    return x


def hash_values(x, w: int, seed: int):
    """Low w bytes of splitmix64(x ^ seed), as the signed integer dtype of width w."""
    import torch
    z = splitmix64(x ^ seed)
    if w == 8:
        return z
    z = z & ((1 << (8 * w)) - 1)
    z = z - ((z >> (8 * w - 1)) & 1) * (1 << (8 * w))      # to signed
    return z.to({1: torch.int8, 2: torch.int16, 4: torch.int32}[w])


def _dtype(w: int):
    import torch
    return {1: torch.int8, 2: torch.int16, 4: torch.int32, 8: torch.int64}[w]


def fill(spec, w: int, seed: int, out=None, device="cuda", h0: int = 0, n: Optional[int] = None,
         chunk: int = 1 << 26):
    """src[h] = H(x(h)) for h in [h0, h0 + n) (default: the whole packed buffer)."""
    import torch
    cols = spec_cols(spec)
    if n is None:
        n = (1 << len(cols)) - h0
    if out is None:
        out = torch.empty(n, dtype=_dtype(w), device=device)
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        h = torch.arange(h0 + s, h0 + e, dtype=torch.int64, device=out.device)
        out[s:e] = hash_values(logical_index(cols, h), w, seed)
    return out


def check(spec, w: int, seed: int, buf, h0: int = 0, chunk: int = 1 << 26) -> int:
    """Number of h in [h0, h0 + buf.numel()) with buf[h] != H(x(h)) under `spec`
    (0 = every element equals the closed form)."""
    import torch
    cols = spec_cols(spec)
    n = buf.numel()
    bad = 0
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        h = torch.arange(h0 + s, h0 + e, dtype=torch.int64, device=buf.device)
        want = hash_values(logical_index(cols, h), w, seed)
        bad += int((buf[s:e].view(want.dtype) != want).sum().item())
    return bad
