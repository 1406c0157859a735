"""Seeded generators for test/bench inputs (no layout arithmetic; see __init__).

Random layouts are returned as literal specs (the same format as configs.py) so
both the oracle and the product ingest them through their own constructors.
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

import numpy as np


def _names(out_dims) -> List[str]:
    """All logical bits, lowest flat bit first (last out dim is fastest)."""
    bits = []
    for name, nb in reversed(list(out_dims)):
        bits += [f"{name}{k}" for k in range(nb)]
    return bits


def random_distributed(rng: np.random.Generator, out_dims, hw_dims: Sequence[Tuple[str, int]],
                       zero_ok: Optional[Sequence[str]] = None):
    """R1: a uniformly random injective assignment of the d logical unit vectors to d
    of the hardware bits; remaining hardware bits are zero (broadcast) columns.
    ``zero_ok`` restricts which hardware dims may receive zero columns (default: any).
    Distributed by construction (Def 4.10)."""
    logical = _names(out_dims)
    slots = [(n, k) for n, nb in hw_dims for k in range(nb)]
    assert len(slots) >= len(logical)
    if zero_ok is None:
        allowed_zero = list(range(len(slots)))
    else:
        allowed_zero = [i for i, (n, _) in enumerate(slots) if n in zero_ok]
    n_zero = len(slots) - len(logical)
    assert len(allowed_zero) >= n_zero
    zero_idx = set(rng.choice(allowed_zero, size=n_zero, replace=False).tolist()) if n_zero else set()
    free = [i for i in range(len(slots)) if i not in zero_idx]
    perm = rng.permutation(len(logical))
    assign = {}
    for i, s in enumerate(free):
        assign[s] = logical[perm[i]]
    ins = []
    for n, nb in hw_dims:
        ins.append((n, [assign.get(i) for i, (m, k) in enumerate(slots) if m == n]))
    return {"out": [tuple(d) for d in out_dims], "in": ins}


def random_memory_cols(rng: np.random.Generator, d: int, max_mixed: Optional[int] = None) -> List[int]:
    """R2: columns of a random memory layout (Def 4.14): a random permutation of unit
    vectors, then up to floor(d/2) columns get a second, strictly lower logical bit.
    Every column keeps a distinct highest bit, so the matrix is invertible by
    construction; columns have 1 or 2 set bits."""
    perm = rng.permutation(d)
    cols = [1 << int(p) for p in perm]
    k = d // 2 if max_mixed is None else min(max_mixed, d // 2)
    chosen = rng.choice(d, size=k, replace=False) if k else []
    for c in chosen:
        top = int(perm[c])
        if top > 0:
            cols[c] |= 1 << int(rng.integers(0, top))
    return cols


def random_surjective_cols(rng: np.random.Generator, d_out: int, d_in: int) -> List[int]:
    """R3: columns of a random surjective F2 matrix (d_out x d_in, d_in >= d_out):
    d_out columns with distinct random highest bits (full rank by construction) plus
    uniform random columns, in random positions."""
    assert d_in >= d_out
    tops = rng.permutation(d_out)
    cols = []
    for t in tops:
        t = int(t)
        low = int(rng.integers(0, 1 << t)) if t > 0 else 0
        cols.append((1 << t) | low)
    for _ in range(d_in - d_out):
        cols.append(int(rng.integers(0, 1 << d_out)))
    order = rng.permutation(d_in)
    return [cols[i] for i in order]


def random_bits(rng: np.random.Generator, n: int, elem_bytes: int) -> np.ndarray:
    """Random bit patterns (NaNs and denormals included when viewed as floats)."""
    dt = {1: np.uint8, 2: np.uint16, 4: np.uint32, 8: np.uint64}[elem_bytes]
    return rng.integers(0, np.iinfo(dt).max, size=n, dtype=dt, endpoint=True)


def splitmix64(x: np.ndarray, seed: int) -> np.ndarray:
    """Hash H(x) for closed-form checks at scale."""
    z = (np.asarray(x, dtype=np.uint64) ^ np.uint64(seed)) + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def random_broadcast_pair(rng: np.random.Generator, n_zero: int, ki: int = 5, kj: int = 5,
                          batch_bits: int = 0, w_bits_a: Optional[Tuple[int, int]] = None,
                          permute_batch: bool = False):
    """Broadcast sweep (P:306-308 zero columns; rule (2) P:358-362): a random bijective
    distributed A and a random distributed B with `n_zero` zero (broadcast) columns over
    reg / lane / warp, on the logical [2^ki, 2^kj] tile, plus `batch_bits` batch bits
    that are the block bits of both (independent tiles) — or, with permute_batch, B's
    block bits a random permutation of A's (a CTA-class map).  Returns (spec_A, spec_B)."""
    d = ki + kj
    out = [("i", ki), ("j", kj)]
    ra = int(rng.integers(1, 4)) if w_bits_a is None else w_bits_a[0]
    wa = d - 5 - ra
    assert wa >= 0
    tot_b = d + n_zero
    rb = int(rng.integers(1, min(6, tot_b - 5) + 1))
    wb = tot_b - 5 - rb
    if wb > 5:
        rb += wb - 5
        wb = 5
    sa = random_distributed(rng, out, [("reg", ra), ("lane", 5), ("warp", wa)])
    sb = random_distributed(rng, out, [("reg", rb), ("lane", 5), ("warp", wb)])
    if batch_bits:
        perm = rng.permutation(batch_bits) if permute_batch else np.arange(batch_bits)
        for s, order in ((sa, np.arange(batch_bits)), (sb, perm)):
            s["out"] = [("b", batch_bits)] + list(s["out"])
            s["in"] = list(s["in"]) + [("block", [f"b{int(k)}" for k in order])]
    return sa, sb
