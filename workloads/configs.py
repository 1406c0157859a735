"""Literal layout tables for the five BASELINE.json configs.

Each layout is written as: output dims (logical, row-major, last fastest — P:142)
and, for every input dim in declaration order (first = least significant hardware
bits — P:138), the logical bit each hardware bit carries ("j3" = bit 3 of dim j,
None = a zero / broadcast column).  These are data, not arithmetic.
"""
from __future__ import annotations

import re
from typing import Dict, List, Optional, Sequence, Tuple

_BIT = re.compile(r"^([A-Za-z_]+)(\d+)$")


def bit_coords(out_dims: Sequence[Tuple[str, int]], bit: Optional[str]) -> Tuple[int, ...]:
    """'j3' -> coordinate tuple with 8 in dim j and 0 elsewhere; None -> zeros."""
    coords = [0] * len(out_dims)
    if bit is None:
        return tuple(coords)
    m = _BIT.match(bit)
    assert m, bit
    name, k = m.group(1), int(m.group(2))
    names = [n for n, _ in out_dims]
    d = names.index(name)
    assert k < out_dims[d][1], (bit, out_dims)
    coords[d] = 1 << k
    return tuple(coords)


def spec_to_bases(spec) -> Tuple[List[Tuple[str, int]], List[Tuple[str, int]], Dict[str, List[Tuple[int, ...]]]]:
    """(in_dims, out_dims, bases) from a literal spec."""
    out_dims = [(n, int(b)) for n, b in spec["out"]]
    in_dims, bases = [], {}
    for name, bits in spec["in"]:
        in_dims.append((name, len(bits)))
        bases[name] = [bit_coords(out_dims, b) for b in bits]
    return in_dims, out_dims, bases


def _b(prefix: str, lo: int, hi: int) -> List[str]:
    return [f"{prefix}{k}" for k in range(lo, hi)]


def _spec(out, reg, lane=None, warp=None, block=None, dev=None, offset=None):
    ins = []
    if offset is not None:
        ins.append(("offset", offset))
    if reg is not None:
        ins.append(("reg", reg))
    if lane is not None:
        ins.append(("lane", lane))
    if warp is not None:
        ins.append(("warp", warp))
    if block is not None:
        ins.append(("block", block))
    if dev is not None:
        ins.append(("dev", dev))
    return {"out": out, "in": ins}


# ---- config 1: Fig. 1, 16x16 fp32, 2 warps (B per G1) ----
C1_OUT = [("i", 4), ("j", 4)]
C1_A = _spec(C1_OUT, ["j0", "i0"], ["j1", "j2", "j3", "i1", "i2"], ["i3"])
C1_B = _spec(C1_OUT, ["i0", "j0"], ["i1", "i2", "i3", "j1", "j2"], ["j3"])


def c1_batched(nb: int):
    out = [("b", nb)] + C1_OUT
    A = _spec(out, ["j0", "i0"], ["j1", "j2", "j3", "i1", "i2"], ["i3"], _b("b", 0, nb))
    B = _spec(out, ["i0", "j0"], ["i1", "i2", "i3", "j1", "j2"], ["j3"], _b("b", 0, nb))
    return A, B


# ---- config 2: wgmma m64n128 accumulator (x2 m-reps) -> blocked [8,8]/[2,16]/[4,1] ----
def c2(nb: int = 16):
    out = [("b", nb), ("i", 7), ("j", 7)]
    A = _spec(out, ["j0", "i3", "j3", "j4", "j5", "j6", "i6"], ["j1", "j2", "i0", "i1", "i2"],
              ["i4", "i5"], _b("b", 0, nb))
    B = _spec(out, ["j0", "j1", "j2", "i0", "i1", "i2", "i6"], ["j3", "j4", "j5", "j6", "i3"],
              ["i4", "i5"], _b("b", 0, nb))
    return A, B


# ---- config 3: 256x128 fp16, blocked row-order -> blocked column-order via smem ----
def c3(nb: int = 14):
    out = [("b", nb), ("i", 8), ("j", 7)]
    A = _spec(out, ["j0", "j1", "j2", "i3", "i4", "i5", "i6", "i7"], ["j3", "j4", "j5", "j6", "i0"],
              ["i1", "i2"], _b("b", 0, nb))
    B = _spec(out, ["i0", "i1", "i2", "j2", "j3", "j4", "j5", "j6"], ["i3", "i4", "i5", "i6", "i7"],
              ["j0", "j1"], _b("b", 0, nb))
    return A, B


def c3b(nb: int = 14):
    out = [("b", nb), ("i", 8), ("j", 7)]
    A = _spec(out, ["j0", "j1", "j2", "i0", "i1", "i2", "i6", "i7"], ["j3", "j4", "j5", "j6", "i3"],
              ["i4", "i5"], _b("b", 0, nb))
    B = _spec(out, ["i0", "i1", "i2", "j0", "j1", "j2", "j5", "j6"], ["i3", "i4", "i5", "i6", "i7"],
              ["j3", "j4"], _b("b", 0, nb))
    return A, B


# ---- config 4: gather / reduce on 4096x4096 fp32 (tiles [128,32] / [128,128]) ----
def c4(kind: str, family: str, n_i: int = 12, n_j: int = 12, k_bits: int = 5):
    """kind in {gather, reduce}; family in {mma, blocked}.  Block bits are the tile
    coordinates: i7.. then j<K>.. (gather, K = 2^k_bits = 16/32/64) / j7.. (reduce)."""
    out = [("i", n_i), ("j", n_j)]
    if kind == "gather":
        jt = k_bits
        if family == "mma":
            # mma accumulator tile [128, K], 4 warps along M: n-reps j3.. then m-rep i6
            reg = ["j0", "i3"] + _b("j", 3, k_bits) + ["i6"]
            lane, warp = ["j1", "j2", "i0", "i1", "i2"], ["i4", "i5"]
        else:
            # blocked [1,4]/[4,8]/[4,1] on [128, K]: lanes j2..j4 (8 along j) when K >= 32
            if k_bits >= 5:
                reg = ["j0", "j1"] + _b("j", 5, k_bits) + ["i4", "i5", "i6"]
                lane, warp = ["j2", "j3", "j4", "i0", "i1"], ["i2", "i3"]
            else:   # K = 16: threads [8, 4]
                reg = ["j0", "j1", "i5", "i6"]
                lane, warp = ["j2", "j3", "i0", "i1", "i2"], ["i3", "i4"]
    else:
        jt = 7
        if family == "mma":
            reg = ["j0", "i3", "j3", "j4", "j5", "j6", "i6"]
            lane, warp = ["j1", "j2", "i0", "i1", "i2"], ["i4", "i5"]
        else:
            reg = ["j0", "j1", "j5", "j6", "i4", "i5", "i6"]
            lane, warp = ["j2", "j3", "j4", "i0", "i1"], ["i2", "i3"]
    block = _b("i", 7, n_i) + _b("j", jt, n_j)
    return _spec(out, reg, lane, warp, block)


# ---- config 5: 32K x 32K bf16 row-sharded -> column-sharded over P = 2^p devices ----
def c5(p: int, n: int = 15):
    out = [("i", n), ("j", n)]
    A = _spec(out, None, offset=_b("j", 0, n) + _b("i", 0, n - p), dev=_b("i", n - p, n))
    B = _spec(out, None, offset=_b("j", 0, n - p) + _b("i", 0, n), dev=_b("j", n - p, n))
    # drop the empty reg entry
    A["in"] = [d for d in A["in"] if d[0] != "reg"]
    B["in"] = [d for d in B["in"] if d[0] != "reg"]
    return A, B


def c5T(p: int, n: int = 15):
    """Variant 5-T: B stores its column shard column-major (offset i fastest)."""
    out = [("i", n), ("j", n)]
    A = {"out": out, "in": [("offset", _b("j", 0, n) + _b("i", 0, n - p)), ("dev", _b("i", n - p, n))]}
    B = {"out": out, "in": [("offset", _b("i", 0, n) + _b("j", 0, n - p)), ("dev", _b("j", n - p, n))]}
    return A, B


CONFIGS = {
    "c1": {"A": C1_A, "B": C1_B, "elem_bytes": 4, "dtype": "f32"},
    "c2": {"A": c2()[0], "B": c2()[1], "elem_bytes": 2, "dtype": "bf16"},
    "c3": {"A": c3()[0], "B": c3()[1], "elem_bytes": 2, "dtype": "f16"},
    "c3b": {"A": c3b()[0], "B": c3b()[1], "elem_bytes": 2, "dtype": "f16"},
}


# ---- §8(f) N1: HBM operand pre-shuffle ----
def n1_preshuffle(kb: int = 12, nb: int = 12):
    """A bf16 weight W[K, N] (K = 2^kb, N = 2^nb) stored row-major (A), rewritten in
    HBM into the packed fragment order of the mma m16n8k16 rhs operand (B; Prop 9.2,
    P:676) for 64 x 32 tiles (4 k-steps, 4 warps along N): every thread's 8 bf16 of
    a tile become one contiguous 16-byte vector."""
    out = [("k", kb), ("n", nb)]
    A = {"out": out, "in": [("offset", _b("n", 0, nb) + _b("k", 0, kb))]}
    B = _spec(out, ["k0", "k3", "k4", "k5"], ["k1", "k2", "n0", "n1", "n2"], ["n3", "n4"],
              _b("k", 6, kb) + _b("n", 5, nb))
    return A, B


# ---- §8(f) N2: tcgen05 TMEM 32x32b accumulator fragment -> coalesced blocked ----
def n2_tmem_epilogue(nb: int = 13):
    """A batch of 2^nb 128 x 128 fp32 accumulator tiles as loaded from TMEM by
    tcgen05.ld.32x32b (thread t of warp w holds row 32w + t; register r column r)
    converted to the blocked [1,4]/[2,16]/[4,1] row-major layout a coalesced epilogue
    store wants."""
    out = [("b", nb), ("i", 7), ("j", 7)]
    A = _spec(out, _b("j", 0, 7), _b("i", 0, 5), ["i5", "i6"], _b("b", 0, nb))
    B = _spec(out, ["j0", "j1", "j6", "i3", "i4", "i5", "i6"], ["j2", "j3", "j4", "j5", "i0"], ["i1", "i2"],
              _b("b", 0, nb))
    return A, B


# ---- §8(f) N2: the other tcgen05.ld fragment shapes (CUTLASS SM100 TMEM_LOAD traits) ----
N2_TMEM_FRAGMENTS = {
    # shape: (reg, lane, warp) logical bits of a 128 x 128 fp32 accumulator tile
    "32x32b": (_b("j", 0, 7), _b("i", 0, 5), ["i5", "i6"]),
    "16x64b": (_b("j", 1, 7) + ["i4"], ["i3", "j0", "i0", "i1", "i2"], ["i5", "i6"]),
    "16x128b": (["i3"] + _b("j", 2, 7) + ["i4"], ["j0", "j1", "i0", "i1", "i2"], ["i5", "i6"]),
    "16x256b": (["j0", "i3"] + _b("j", 3, 7) + ["i4"], ["j1", "j2", "i0", "i1", "i2"], ["i5", "i6"]),
}


def n2_tmem(shape: str, nb: int = 13):
    """A batch of 2^nb 128 x 128 fp32 accumulator tiles as loaded from TMEM by
    tcgen05.ld.<shape> (N2_TMEM_FRAGMENTS) converted to the coalesced blocked
    [1,4]/[2,16]/[4,1] row-major epilogue layout (as n2_tmem_epilogue)."""
    reg, lane, warp = N2_TMEM_FRAGMENTS[shape]
    out = [("b", nb), ("i", 7), ("j", 7)]
    A = _spec(out, reg, lane, warp, _b("b", 0, nb))
    B = n2_tmem_epilogue(nb)[1]
    return A, B


def n2_acc_to_lhs(bits: int, nb: int = 14):
    """Chained GEMM (P:28 FlashAttention's register reuse; Prop 9.2): a batch
    of 2^nb 64 x 64 wgmma m64n64 accumulator tiles (4 warps along M; G17), downcast to
    `bits`-bit elements, converted into the register-A (lhs) operand of the next wgmma
    (m64nNk{32/bits*8}).  bf16 (16): the two layouts coincide (NOOP).  fp8 (8): the lhs
    holds 4 consecutive k per register, so k bits 1 and 3 swap between a register and
    a lane — an intra-warp shuffle."""
    out = [("b", nb), ("i", 6), ("j", 6)]
    A = _spec(out, ["j0", "i3", "j3", "j4", "j5"], ["j1", "j2", "i0", "i1", "i2"], ["i4", "i5"], _b("b", 0, nb))
    if bits == 16:
        B = _spec(out, ["j0", "i3", "j3", "j4", "j5"], ["j1", "j2", "i0", "i1", "i2"], ["i4", "i5"], _b("b", 0, nb))
    elif bits == 8:
        B = _spec(out, ["j0", "j1", "i3", "j4", "j5"], ["j2", "j3", "i0", "i1", "i2"], ["i4", "i5"], _b("b", 0, nb))
    else:
        raise ValueError(bits)
    return A, B


# ---- §8(e)(2): partial device exchanges (a dev bit shared by A and B) ----
def c5_partial(p: int, n: int = 15, swap: bool = False):
    """Config 5 with the top row bit i_{n-1} a device bit of BOTH layouts (p >= 2): A is
    row-sharded over (i_{n-p} .. i_{n-1}); B moves the low p-1 of those rows into its
    offset and shards its columns j_{n-p+1} .. j_{n-1} instead, keeping i_{n-1} as a dev
    bit — at the same position (rank bit p-1) or, with swap, as rank bit 0.  Each rank
    then exchanges with 2^(p-1) ranks, not 2^p: a partial exchange."""
    assert p >= 2
    out = [("i", n), ("j", n)]
    A = {"out": out, "in": [("offset", _b("j", 0, n) + _b("i", 0, n - p)), ("dev", _b("i", n - p, n))]}
    jdev = _b("j", n - p + 1, n)
    bdev = (["i" + str(n - 1)] + jdev) if swap else (jdev + ["i" + str(n - 1)])
    B = {"out": out, "in": [("offset", _b("j", 0, n - p + 1) + _b("i", 0, n - 1)), ("dev", bdev)]}
    return A, B
