"""CPU ORACLE for the Linear Layouts conversion hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import or call anything in this file.  The product
(``paper_conf_asplos_0001cgrnls0trm26_b200``) never imports it and shares no code,
header, table or helper with it; the only module both sides use is ``workloads``
(seeded input generators and literal basis tables, no layout arithmetic).

Everything here is a plain, slow, obviously-correct restatement of
"Linear Layouts: Robust Code Generation of Efficient Tensor Computation Using F2"
(ASPLOS '26).  Citations ``P:L`` are line numbers of /root/reference/PAPER.md
(section / definition given beside them).  Readings of garbled or silent passages
follow SURVEY.md §8(c) (G1..G23) and are listed in DESIGN.md §3.

Conventions:
* a layout maps labelled input (hardware) bits to labelled output (logical) bits;
  ``basis[k]`` is the tuple of output coordinates hit by input bit k;
* the *hardware flat index* h concatenates input dims in declaration order, the
  first declared dim least significant ("the first 2 bits represent Reg",
  P:148 footnote "least significant bits come first");
* the *logical flat index* is row-major over the output dims in declaration order,
  the last dim fastest ("j is the fastest moving dimension");
* a buffer "packed in layout L" holds at position h the logical element L(h).

Every function that has no independent pin says so in its docstring
("parity unpinned"); see tests/test_oracle_*.py for the pins.
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass, field
from typing import Dict, List, Sequence, Tuple

import numpy as np

# --------------------------------------------------------------------------------------
# O1  Representation  (Def 4.1 "a linear map between labeled vector spaces")
# --------------------------------------------------------------------------------------

LEVEL_OF_DIM = {  # hardware hierarchy used by the class oracle (O7)
    "reg": 0, "register": 0,
    "lane": 1, "thr": 1, "thread": 1,
    "warp": 2, "wrp": 2,
    "block": 3, "cta": 3, "offset": 3,
    "dev": 4, "device": 4,
}
CLASS_OF_LEVEL = {0: "REGPERM", 1: "SHUFFLE", 2: "SMEM", 3: "CTA", 4: "DEVICE"}


def logical_flat(out_dims: Sequence[Tuple[str, int]], coords: Sequence[int]) -> int:
    """Row-major flat index over the output dims, last dim fastest."""
    assert len(coords) == len(out_dims)
    flat = 0
    for (name, nbits), c in zip(out_dims, coords):
        c = int(c)
        assert 0 <= c < (1 << nbits), (name, c)
        flat = (flat << nbits) | c
    return flat


def logical_coords(out_dims: Sequence[Tuple[str, int]], flat: int) -> Tuple[int, ...]:
    """Inverse of :func:`logical_flat`."""
    coords = []
    for name, nbits in reversed(list(out_dims)):
        coords.append(flat & ((1 << nbits) - 1))
        flat >>= nbits
    return tuple(reversed(coords))


def hw_flat(in_dims: Sequence[Tuple[str, int]], coords: Sequence[int]) -> int:
    """Hardware flat index: first declared dim least significant."""
    h, shift = 0, 0
    for (name, nbits), c in zip(in_dims, coords):
        assert 0 <= int(c) < (1 << nbits), (name, c)
        h |= int(c) << shift
        shift += nbits
    return h


def hw_coords(in_dims: Sequence[Tuple[str, int]], h: int) -> Tuple[int, ...]:
    """Inverse of :func:`hw_flat`."""
    out = []
    for name, nbits in in_dims:
        out.append(h & ((1 << nbits) - 1))
        h >>= nbits
    return tuple(out)


@dataclass
class Layout:
    """A linear layout between labelled F2 spaces (Def 4.1).

    ``bases[name]`` lists, for every bit of input dim ``name`` (bit 0 first), the
    output coordinates that bit maps to.  ``cols`` is the same information as
    logical flat indices, one per input bit in hardware-flat order (the matrix
    columns of P:140).
    """
    in_dims: List[Tuple[str, int]]
    out_dims: List[Tuple[str, int]]
    bases: Dict[str, List[Tuple[int, ...]]]
    cols: List[int] = field(init=False)

    def __post_init__(self):
        self.in_dims = [(str(n), int(b)) for n, b in self.in_dims]
        self.out_dims = [(str(n), int(b)) for n, b in self.out_dims]
        self.cols = []
        for name, nbits in self.in_dims:
            vecs = self.bases.get(name, [])
            assert len(vecs) == nbits, f"dim {name}: {len(vecs)} basis vectors for {nbits} bits"
            for v in vecs:
                self.cols.append(logical_flat(self.out_dims, tuple(v)))

    @property
    def d_in(self) -> int:
        return sum(b for _, b in self.in_dims)

    @property
    def d_out(self) -> int:
        return sum(b for _, b in self.out_dims)

    def dim_bits(self, name: str) -> List[int]:
        """Hardware-flat bit positions that belong to input dim ``name``."""
        pos = 0
        for n, b in self.in_dims:
            if n == name:
                return list(range(pos, pos + b))
            pos += b
        return []

    def cols_of(self, name: str) -> List[int]:
        """The columns L_name of P:352 (logical flats of the bits of dim ``name``)."""
        return [self.cols[k] for k in self.dim_bits(name)]


def layout_from_cols(in_dims, out_dims, cols: Sequence[int]) -> Layout:
    """Build a Layout from logical-flat columns listed in hardware-flat bit order."""
    bases, k = {}, 0
    for name, nbits in in_dims:
        bases[name] = [logical_coords(out_dims, int(cols[k + i])) for i in range(nbits)]
        k += nbits
    return Layout(list(in_dims), list(out_dims), bases)


# --------------------------------------------------------------------------------------
# O2  Apply  ("Bitwise XOR of these three coordinate pairs yields the
#              register's absolute position"; w = Av over F2)
# --------------------------------------------------------------------------------------

def apply(L: Layout, h: int) -> int:
    """L(h) for one hardware flat index h: XOR of the columns of the set bits."""
    x = 0
    for k, c in enumerate(L.cols):
        if (h >> k) & 1:
            x ^= c
    return x


def apply_all(L: Layout, hs: np.ndarray) -> np.ndarray:
    """Vectorised :func:`apply` over an array of hardware flat indices (bit by bit)."""
    hs = np.asarray(hs, dtype=np.uint64)
    x = np.zeros(hs.shape, dtype=np.uint64)
    for k, c in enumerate(L.cols):
        bit = (hs >> np.uint64(k)) & np.uint64(1)
        x ^= bit * np.uint64(c)
    return x


def image_table(L: Layout) -> np.ndarray:
    """L(h) for every h in [0, 2^d_in) (enumeration; small layouts only)."""
    assert L.d_in <= 26, "enumeration only for small layouts"
    return apply_all(L, np.arange(1 << L.d_in, dtype=np.uint64))


# --------------------------------------------------------------------------------------
# O3  Predicates by enumeration  (Def 4.5, Def 4.10, Def 4.14 P:276,
#      Remark P:224)
# --------------------------------------------------------------------------------------

def is_surjective(L: Layout) -> bool:
    return len(np.unique(image_table(L))) == (1 << L.d_out)


def is_injective(L: Layout) -> bool:
    return len(np.unique(image_table(L))) == (1 << L.d_in)


def is_distributed(L: Layout) -> bool:
    """Def 4.10: surjective, each column has at most one set bit, no repeated
    non-zero columns."""
    nz = [c for c in L.cols if c != 0]
    return (is_surjective(L)
            and all(bin(c).count("1") <= 1 for c in L.cols)
            and len(set(nz)) == len(nz))


def is_memory(L: Layout) -> bool:
    """Def 4.14: invertible, every column has 1 or 2 set bits."""
    return (L.d_in == L.d_out and is_surjective(L)
            and all(1 <= bin(c).count("1") <= 2 for c in L.cols))


# --------------------------------------------------------------------------------------
# O4  Preimages and the right inverse  (Def 4.5; slack = 0)
# --------------------------------------------------------------------------------------

def preimage_min(L: Layout) -> np.ndarray:
    """first[x] = min{h : L(h) = x}, by scanning h in ascending order (brute force).

    Raises if L is not surjective (a right inverse exists only then)."""
    img = image_table(L)
    xs, first = np.unique(img, return_index=True)   # index of the first occurrence
    if len(xs) != (1 << L.d_out):
        raise ValueError("layout is not surjective; no right inverse (P:194)")
    table = np.empty(1 << L.d_out, dtype=np.int64)
    table[xs.astype(np.int64)] = first
    return table


def right_inverse_cols(L: Layout) -> List[int]:
    """Solve M X = I over F2 by Gaussian elimination, free variables set to 0
    (the "slack variables ... set to zeros" of P:362).  Pivots are taken over the
    columns of M in ascending order.  Returns, for every logical bit t (flat bit
    order, bit 0 = lowest logical flat bit), the hardware flat index X e_t."""
    pivots: Dict[int, Tuple[int, int]] = {}   # leading logical bit -> (vector, combination)
    for k, c in enumerate(L.cols):
        v, comb = c, 1 << k
        while v:
            lead = v.bit_length() - 1
            if lead not in pivots:
                pivots[lead] = (v, comb)
                break
            pv, pc = pivots[lead]
            v ^= pv
            comb ^= pc
        # v == 0: column k depends on earlier columns -> a free variable, kept at 0
    if len(pivots) != L.d_out:
        raise ValueError("layout is not surjective; no right inverse (P:194)")
    out = []
    for t in range(L.d_out):
        v, comb = 1 << t, 0
        while v:
            lead = v.bit_length() - 1
            pv, pc = pivots[lead]
            v ^= pv
            comb ^= pc
        out.append(comb)
    return out


def right_inverse(L: Layout) -> Layout:
    """The right inverse as a layout from the logical space back to hardware:
    its input dims are L's output dims and its output dims are L's input dims."""
    hcols = right_inverse_cols(L)          # per logical flat bit (lowest first)
    # logical flat bit order is: last out dim's bits first (it is the fastest)
    per_bit = {}
    pos = 0
    for name, nbits in reversed(L.out_dims):
        per_bit[name] = hcols[pos:pos + nbits]
        pos += nbits
    bases = {name: [hw_coords(L.in_dims, h) for h in per_bit[name]] for name, _ in L.out_dims}
    # out dims of the inverse are L's in dims; its "logical" coordinates are hw coords
    return Layout(list(L.out_dims), list(L.in_dims), bases)


def apply_inverse_all(L: Layout, xs: np.ndarray) -> np.ndarray:
    """h = L^{-1}(x) (slack-zero right inverse) for logical flat indices xs."""
    hcols = right_inverse_cols(L)
    xs = np.asarray(xs, dtype=np.uint64)
    h = np.zeros(xs.shape, dtype=np.uint64)
    for t, hc in enumerate(hcols):
        h ^= ((xs >> np.uint64(t)) & np.uint64(1)) * np.uint64(hc)
    return h


# --------------------------------------------------------------------------------------
# O6  Composition, product, left division  (Defs 4.2-4.4)
# --------------------------------------------------------------------------------------

def apply_coords(L: Layout, in_coords: Sequence[int]) -> Tuple[int, ...]:
    return logical_coords(L.out_dims, apply(L, hw_flat(L.in_dims, in_coords)))


def compose(L2: Layout, L1: Layout) -> Layout:
    """L2 ∘ L1 : u -> L2(L1(u))  (Def 4.2).  Requires L1.out == L2.in."""
    if L1.out_dims != L2.in_dims:
        raise ValueError("dimension mismatch: L1.out_dims != L2.in_dims")
    bases = {}
    for name, nbits in L1.in_dims:
        bases[name] = [apply_coords(L2, v) for v in L1.bases[name]]
    return Layout(list(L1.in_dims), list(L2.out_dims), bases)


def product(L1: Layout, L2: Layout) -> Layout:
    """L1 × L2 (Def 4.3), label-wise: dims with the same name are
    concatenated with L1's bits low; L2's images are shifted above L1's range."""
    def merge(d1, d2):
        names = [n for n, _ in d1] + [n for n, _ in d2 if n not in dict(d1)]
        s1, s2 = dict(d1), dict(d2)
        return [(n, s1.get(n, 0) + s2.get(n, 0)) for n in names]
    in_dims = merge(L1.in_dims, L2.in_dims)
    out_dims = merge(L1.out_dims, L2.out_dims)
    o1 = dict(L1.out_dims)
    bases = {n: [] for n, _ in in_dims}
    for n, _ in in_dims:
        for v in L1.bases.get(n, []):
            c1 = dict(zip([d for d, _ in L1.out_dims], v))
            bases[n].append(tuple(c1.get(d, 0) for d, _ in out_dims))
        for v in L2.bases.get(n, []):
            c2 = dict(zip([d for d, _ in L2.out_dims], v))
            bases[n].append(tuple(c2.get(d, 0) << o1.get(d, 0) for d, _ in out_dims))
    return Layout(in_dims, out_dims, bases)


def left_divide(M: Layout, M1: Layout) -> Layout:
    """M /_l M1 = M2 iff M = diag(M1, M2) label-wise (Def 4.4).

    For each input dim of M1: M's low bits of that dim must reproduce M1, and M's
    remaining bits must map to zero in M1's output range.  Raises if not divisible."""
    mo = dict(M.out_dims)
    m1o = dict(M1.out_dims)
    m1i = dict(M1.in_dims)
    out_names = [n for n, _ in M.out_dims]
    in_dims2 = [(n, b - m1i.get(n, 0)) for n, b in M.in_dims]
    out_dims2 = [(n, mo[n] - m1o.get(n, 0)) for n in out_names]
    if any(b < 0 for _, b in in_dims2 + out_dims2):
        raise ValueError("not divisible: M1 larger than M")
    bases2 = {}
    for n, b in M.in_dims:
        vecs = M.bases[n]
        k1 = m1i.get(n, 0)
        for i in range(k1):
            c1 = dict(zip([d for d, _ in M1.out_dims], M1.bases[n][i]))
            want = tuple(c1.get(d, 0) for d in out_names)
            if tuple(vecs[i]) != want:
                raise ValueError(f"not divisible: dim {n} bit {i}")
        rest = []
        for v in vecs[k1:]:
            cv = dict(zip(out_names, v))
            for d in out_names:                   # must vanish on M1's output range
                if cv[d] & ((1 << m1o.get(d, 0)) - 1):
                    raise ValueError(f"not divisible: dim {n} overlaps M1's range")
            rest.append(tuple(cv[d] >> m1o.get(d, 0) for d in out_names))
        bases2[n] = rest
    return Layout(in_dims2, out_dims2, bases2)


# --------------------------------------------------------------------------------------
# O5  Conversion  (§5.4; pull form of B^{-1}∘A)
# --------------------------------------------------------------------------------------

def pack(L: Layout, T: np.ndarray) -> np.ndarray:
    """Buffer packed in layout L: pack_L(T)[h] = T[L(h)]."""
    return np.asarray(T).reshape(-1)[image_table(L).astype(np.int64)]


def convert(A: Layout, B: Layout, src: np.ndarray) -> np.ndarray:
    """dst[h] = src[first_A[B(h)]] for every h of B (O5).  Brute-force preimage."""
    if A.out_dims != B.out_dims:
        raise ValueError("A and B must describe the same logical tensor")
    first = preimage_min(A)
    return np.asarray(src).reshape(-1)[first[image_table(B).astype(np.int64)]]


def convert_at(A: Layout, B: Layout, src: np.ndarray, hs: np.ndarray) -> np.ndarray:
    """dst[h] for selected h (large layouts): src[A^{-1}(B(h))] with the slack-zero
    right inverse (equal to the min-index preimage, pinned in the tests)."""
    xs = apply_all(B, hs)
    return np.asarray(src).reshape(-1)[apply_inverse_all(A, xs).astype(np.int64)]


def is_consistent(A: Layout, src: np.ndarray) -> bool:
    """A-consistency of src: A(h1)=A(h2) implies equal elements."""
    img = image_table(A).astype(np.int64)
    first = preimage_min(A)
    s = np.asarray(src).reshape(-1)
    return bool(np.all(s == s[first[img]]))


# --------------------------------------------------------------------------------------
# O7  Class oracle — existential, brute force (P:364-373 and the smem fallback P:391)
# --------------------------------------------------------------------------------------

def _level_coords(L: Layout, hs: np.ndarray, level: int) -> List[np.ndarray]:
    """Coordinates of the input dims whose level is above ``level``, by name."""
    out = {}
    shift = 0
    for name, nbits in L.in_dims:
        if LEVEL_OF_DIM[name] > level:
            out[name] = (hs >> np.uint64(shift)) & np.uint64((1 << nbits) - 1)
        shift += nbits
    return out


def classify(A: Layout, B: Layout) -> str:
    """Lowest level λ such that every dst index h of B has a preimage h' under A of
    B(h) agreeing with h on every input dimension above λ; NOOP iff A(h)=B(h) ∀h."""
    if A.out_dims != B.out_dims:
        raise ValueError("A and B must describe the same logical tensor")
    ha = np.arange(1 << A.d_in, dtype=np.uint64)
    hb = np.arange(1 << B.d_in, dtype=np.uint64)
    xa, xb = apply_all(A, ha), apply_all(B, hb)
    if A.in_dims == B.in_dims and np.array_equal(xa, xb):
        return "NOOP"
    names = sorted({LEVEL_OF_DIM[n] for n, _ in A.in_dims + B.in_dims})
    for level in range(0, 5):
        ca, cb = _level_coords(A, ha, level), _level_coords(B, hb, level)
        keys = sorted(set(ca) | set(cb))
        zeros_a, zeros_b = np.zeros_like(ha), np.zeros_like(hb)
        ka = np.stack([xa] + [ca.get(k, zeros_a) for k in keys], axis=1)
        kb = np.stack([xb] + [cb.get(k, zeros_b) for k in keys], axis=1)
        sa = {tuple(r) for r in ka.tolist()}
        if all(tuple(r) in sa for r in kb.tolist()):
            return CLASS_OF_LEVEL[level]
    raise AssertionError("unreachable: level 4 always succeeds for surjective A")


# --------------------------------------------------------------------------------------
# Layout families (§4.3; Props 9.1 / 9.2 in the appendix)
# --------------------------------------------------------------------------------------

def blocked(shape, size_per_thread, threads_per_warp, warps_per_cta, order,
            block_dims=True) -> Layout:
    """Blocked layout σ_o^{-1}∘(id_R^o × id_T^o × id_W^o) (Prop 9.1).

    Registers take the sizePerThread bits in ``order`` (fastest dim first), then
    lanes, then warps; when the CTA tile is smaller than ``shape`` the remaining bits
    of each dim (in ``order``) become further register bits (Triton's repetition,
    SURVEY Appendix A notes); when it is larger, the excess bits map to zero
    (broadcast).  Output dims are named ``d0, d1, ...``; flat bit order is
    row-major."""
    nd = len(shape)
    lg = lambda v: int(v).bit_length() - 1
    sb = [lg(s) for s in shape]
    used = [0] * nd
    def take(count_per_dim):
        vecs = []
        for d in order:
            for _ in range(lg(count_per_dim[d])):
                c = [0] * nd
                if used[d] < sb[d]:
                    c[d] = 1 << used[d]
                used[d] += 1
                vecs.append(tuple(c))
        return vecs
    reg = take(size_per_thread)
    lane = take(threads_per_warp)
    warp = take(warps_per_cta)
    for d in order:                         # repetitions -> more registers
        while used[d] < sb[d]:
            c = [0] * nd
            c[d] = 1 << used[d]
            used[d] += 1
            reg.append(tuple(c))
    out_dims = [(f"d{i}", sb[i]) for i in range(nd)]
    in_dims = [("reg", len(reg)), ("lane", len(lane)), ("warp", len(warp))]
    return Layout(in_dims, out_dims, {"reg": reg, "lane": lane, "warp": warp})


def mma_acc(shape, warps_m, warps_n=1) -> Layout:
    """Accumulator (output) tile of mma m16n8 / wgmma (Prop 9.2, G17):
    reg0→j0, lanes (j1, j2, i0, i1, i2), reg1→i3; warps along M first, then
    N; repetitions as register bits, n-repetitions before m-repetitions."""
    M, N = shape
    lg = lambda v: int(v).bit_length() - 1
    mb, nb = lg(M), lg(N)
    I = lambda k: (1 << k, 0) if k < mb else (0, 0)
    J = lambda k: (0, 1 << k) if k < nb else (0, 0)
    reg = [J(0), I(3)]
    lane = [J(1), J(2), I(0), I(1), I(2)]
    wm, wn = lg(warps_m), lg(warps_n)
    warp = [I(4 + k) for k in range(wm)] + [J(3 + k) for k in range(wn)]
    for k in range(3 + wn, nb):              # n repetitions
        reg.append(J(k))
    for k in range(4 + wm, mb):              # m repetitions
        reg.append(I(k))
    in_dims = [("reg", len(reg)), ("lane", 5), ("warp", len(warp))]
    return Layout(in_dims, [("d0", mb), ("d1", nb)], {"reg": reg, "lane": lane, "warp": warp})


def mma_operand(is_rhs: bool, shape, bitwidth: int, warps_m: int = 1, warps_n: int = 1) -> Layout:
    """mma / wgmma input operand tiles (Prop 9.2), written from the paper:
        lhs:  id^{Reg,1}_{log2(32/b)} x id^{Thr,1}_2 x id^{Thr,0}_3 x id^{Reg,0}_1 x id^{Reg,1}_1
        rhs:  id^{Reg,0}_{log2(32/b)} x id^{Thr,0}_2 x id^{Thr,1}_3 x id^{Reg,1}_1
    (the product is taken left to right, each factor's bits above the previous ones in
    its dims).  Dims: lhs (d0 = M, d1 = K), rhs (d0 = K, d1 = N).  Repetitions: over the
    K dim first, then the other dim, as register bits.  Warps: warps_m split M and
    warps_n split N; the operand is broadcast over the other dim's warps
    (zero columns)."""
    rows, cols = shape
    rb, cb = int(rows).bit_length() - 1, int(cols).bit_length() - 1
    kb = (32 // bitwidth).bit_length() - 1
    used = {0: 0, 1: 0}
    def take(dim):
        c = [0, 0]
        nb = rb if dim == 0 else cb
        if used[dim] < nb:
            c[dim] = 1 << used[dim]
        used[dim] += 1
        return tuple(c)
    kdim, odim = (0, 1) if is_rhs else (1, 0)
    reg, lane, warp = [], [], []
    reg += [take(kdim) for _ in range(kb)]
    lane += [take(kdim) for _ in range(2)]
    lane += [take(odim) for _ in range(3)]
    if not is_rhs:
        reg.append(take(odim))
    reg.append(take(kdim))
    wm, wn = int(warps_m).bit_length() - 1, int(warps_n).bit_length() - 1
    for _ in range(wm):
        warp.append((0, 0) if is_rhs else take(odim))
    for _ in range(wn):
        warp.append(take(odim) if is_rhs else (0, 0))
    nbk = rb if is_rhs else cb
    nbo = cb if is_rhs else rb
    while used[kdim] < nbk:
        reg.append(take(kdim))
    while used[odim] < nbo:
        reg.append(take(odim))
    in_dims = [("reg", len(reg)), ("lane", 5), ("warp", len(warp))]
    return Layout(in_dims, [("d0", rb), ("d1", cb)], {"reg": reg, "lane": lane, "warp": warp})


TMEM_SHAPES = ("32x32b", "16x64b", "16x128b", "16x256b")


def tmem_ld(shape: str, M: int, N: int) -> Layout:
    """Registers of a warpgroup after loading a 128 x N fp32 accumulator from Blackwell
    tensor memory (P:53 names tensor memory) with
    tcgen05.ld.sync.aligned.<shape>.x<num>.b32 — TMEM lane (data path) = row i, TMEM
    column (32-bit) = column j [HW]; warp w of the warpgroup reads lanes [32w, 32w+32).
    Per warp and x1 repetition (PTX "matrix fragments for tcgen05.ld"):
      32x32b : thread t <- lane t; 1 register: column 0.
      16x64b : 16 lanes x 2 columns; thread t <- row 8*t0 + (t >> 2), column t1
               (t0, t1 = bits 0, 1 of t); 1 register.
      16x128b: 16 lanes x 4 columns; thread t <- row (t >> 2), column t & 3;
               register r <- row + 8r; 2 registers.
      16x256b: 16 lanes x 8 columns; thread t <- row (t >> 2), column 2*(t & 3) + r0;
               register r = r0 + 2 r1 <- row + 8 r1 (the mma m16n8 C fragment); 4 registers.
    Repetitions .x<num> step along the columns (register bits above the x1 ones, column
    bits above the x1 width, ascending); 16-lane shapes then take a second load 16 lanes
    down (one more register bit -> row bit 4); warps -> rows 5, 6.  Pinned to the CUTLASS
    SM100 TMEM_LOAD copy traits (tests/test_oracle_pins.py)."""
    assert M == 128, "a warpgroup reads 128 TMEM lanes"
    nb = int(N).bit_length() - 1
    I = lambda k: (1 << k, 0)
    J = lambda k: (0, 1 << k) if k < nb else (0, 0)
    if shape == "32x32b":
        reg0, lane, w_cols, rows16 = [], [I(0), I(1), I(2), I(3), I(4)], 0, False
    elif shape == "16x64b":
        reg0, lane, w_cols, rows16 = [], [I(3), J(0), I(0), I(1), I(2)], 1, True
    elif shape == "16x128b":
        reg0, lane, w_cols, rows16 = [I(3)], [J(0), J(1), I(0), I(1), I(2)], 2, True
    elif shape == "16x256b":
        reg0, lane, w_cols, rows16 = [J(0), I(3)], [J(1), J(2), I(0), I(1), I(2)], 3, True
    else:
        raise ValueError(shape)
    assert nb >= w_cols, "N smaller than one x1 load"
    reg = list(reg0) + [J(k) for k in range(w_cols, nb)]
    if rows16:
        reg.append(I(4))
    warp = [I(5), I(6)]
    in_dims = [("reg", len(reg)), ("lane", 5), ("warp", 2)]
    return Layout(in_dims, [("d0", 7), ("d1", nb)], {"reg": reg, "lane": lane, "warp": warp})


def sliced(L: Layout, dim: int) -> Layout:
    """Slice: remove logical dim ``dim`` (Prop 4.8).  The result may be
    non-injective (zero columns) but stays surjective (Remark P:224)."""
    keep = [i for i in range(len(L.out_dims)) if i != dim]
    out_dims = [L.out_dims[i] for i in keep]
    bases = {n: [tuple(v[i] for i in keep) for v in L.bases[n]] for n, _ in L.in_dims}
    return Layout(list(L.in_dims), out_dims, bases)


def mma_swizzle_offset(i: int, j: int, vec: int, per_phase: int, max_phase: int) -> int:
    """Def 4.11, the in-row offset (in elements):
    ((i/per_phase mod max_phase) XOR j/vec)·vec XOR (j mod vec)."""
    return ((((i // per_phase) % max_phase) ^ (j // vec)) * vec) ^ (j % vec)


def mma_swizzle_C(m: int, n: int, vec: int, per_phase: int, max_phase: int) -> List[int]:
    """Rows c_i of C in [[I_n, C], [0, I_m]]:
    c_i = (vec · ((2^i / per_phase) mod max_phase)) mod 2^n."""
    return [(vec * (((1 << i) // per_phase) % max_phase)) % (1 << n) for i in range(m)]


def mma_swizzle_layout(m: int, n: int, vec: int, per_phase: int, max_phase: int) -> Layout:
    """The linear map logical (i, j) -> offset of Def 4.11 written as the matrix
    [[I_n, C], [0, I_m]] of P:260 (full offset = i·2^n + in-row offset, G18).
    Input dims (j, i) low first; output is the offset."""
    C = mma_swizzle_C(m, n, vec, per_phase, max_phase)
    jb = [((1 << k) + 0,) for k in range(n)]                # j bits: identity on low n
    ib = [(((1 << k) << n) | C[k],) for k in range(m)]     # i bits: I_m above, C in low
    return Layout([("j", n), ("i", m)], [("offset", m + n)], {"j": jb, "i": ib})


def identity_memory(out_dims) -> Layout:
    """Unswizzled memory layout: offset -> the same row-major coordinate."""
    d = sum(b for _, b in out_dims)
    cols = [1 << k for k in range(d)]
    return layout_from_cols([("offset", d)], out_dims, cols)


# --------------------------------------------------------------------------------------
# O8  Shared-memory bank model (Lemma 9.4; wavefront split P:406)
# --------------------------------------------------------------------------------------

def smem_wavefronts(S: Layout, L: Layout, w: int, vec_cols: Sequence[int],
                    bank_bytes: int = 4, n_banks: int = 32) -> Tuple[int, int]:
    """Simulate every warp-level vector access of distributed layout L to the
    shared-memory layout S (offset -> logical, bijective) with element size w bytes.

    The vector accessed by one lane is the coset over the logical vectors
    ``vec_cols`` (they must be among L's register columns and S's lowest offset
    bits, in order).  An access of a = 2^v·w bytes per lane is split into phases of
    (n_banks·bank_bytes)/a lanes when a > bank_bytes ("transactions involving
    more than 128 bytes will be split"), otherwise one phase of all lanes.  Per
    phase, wavefronts = max over banks of the number of distinct bank words touched
    (same word = broadcast, not a conflict).  Returns (wavefronts, ideal), ideal =
    bytes / (n_banks·bank_bytes) rounded up per phase."""
    v = len(vec_cols)
    a = (1 << v) * w
    seg_bytes = n_banks * bank_bytes
    lane_bits = L.dim_bits("lane")
    nl = len(lane_bits)
    reg_bits = L.dim_bits("reg")
    warp_bits = L.dim_bits("warp")
    vec_reg_bits = []
    for c in vec_cols:
        ks = [k for k in reg_bits if L.cols[k] == c]
        assert len(ks) == 1, "vector columns must be register columns of L"
        vec_reg_bits.append(ks[0])
    other_reg = [k for k in reg_bits if k not in vec_reg_bits]
    S_inv = preimage_min(S)                   # logical -> offset (S bijective)
    for t, c in enumerate(vec_cols):
        assert S.cols[t] == c, "S_Vec must be the lowest offset bits"
    lanes_per_phase = max(1, min(1 << nl, seg_bytes // a)) if a > bank_bytes else (1 << nl)
    total = ideal = 0
    for wi in range(1 << len(warp_bits)):
        for ri in range(1 << len(other_reg)):
            base = 0
            for t, k in enumerate(warp_bits):
                if (wi >> t) & 1:
                    base |= 1 << k
            for t, k in enumerate(other_reg):
                if (ri >> t) & 1:
                    base |= 1 << k
            byte_addr = []
            for l in range(1 << nl):
                h = base
                for t, k in enumerate(lane_bits):
                    if (l >> t) & 1:
                        h |= 1 << k
                off = int(S_inv[apply(L, h)])
                byte_addr.append(off * w)
            for p0 in range(0, 1 << nl, lanes_per_phase):
                words = set()
                for l in range(p0, p0 + lanes_per_phase):
                    for b in range(0, a, min(a, bank_bytes)):
                        words.add((byte_addr[l] + b) // bank_bytes)
                per_bank: Dict[int, int] = {}
                for wd in words:
                    per_bank[wd % n_banks] = per_bank.get(wd % n_banks, 0) + 1
                total += max(per_bank.values())
                ideal += -(-(lanes_per_phase * a) // seg_bytes)
    return total, ideal


def smem_matrix_wavefronts(S: Layout, L: Layout, w: int, word_cols: Sequence[int],
                           trans: bool = False, bank_bytes: int = 4,
                           n_banks: int = 32) -> Tuple[int, int]:
    """The same bank model for the ldmatrix / stmatrix instructions ("each
    thread ... handle[s] 4 contiguous bytes, with 8 groups of 4 threads collaborating
    to store a row each"; the fragment is PTX's m8n8 b16 matrix [HW]).

    Every thread holds one 32-bit word per matrix, made of the elements over the
    logical vectors ``word_cols`` (the log2(4/w) register columns of L whose elements
    form the word, lowest first).  Non-transposed: lane l's word is bytes 4·(l mod 4)
    .. +3 of row l div 4 of the matrix; transposed (.trans, w = 2): the two halves h
    of lane l's word are column l div 4 of rows 2·(l mod 4) + h.  The matrices are
    enumerated by L's remaining register bits and its warp bits.  Every matrix must
    really be 8 rows of 16 contiguous, 16-byte aligned bytes in S (the instruction
    can lower L, Thm 5.1) — otherwise ValueError.  A matrix takes one
    128-byte wavefront per distinct row in its most loaded 16-byte bank group
    (rows are whole 16-byte pieces of the 128-byte segment).  Returns
    (wavefronts, ideal); ideal = 1 per matrix."""
    if trans and w != 2:
        raise ValueError(".trans moves b16 elements")
    k = (4 // w).bit_length() - 1
    if len(word_cols) != k:
        raise ValueError("a 32-bit word holds 4/w elements")
    lane_bits = L.dim_bits("lane")
    reg_bits = L.dim_bits("reg")
    warp_bits = L.dim_bits("warp")
    word_bits = []
    for c in word_cols:
        ks = [b for b in reg_bits if L.cols[b] == c]
        assert len(ks) == 1, "word columns must be register columns of L"
        word_bits.append(ks[0])
    other = [b for b in reg_bits if b not in word_bits] + list(warp_bits)
    S_inv = preimage_min(S)
    group_bytes = n_banks * bank_bytes // 8        # 16-byte bank groups of a segment
    total = ideal = 0
    for m in range(1 << len(other)):
        base = 0
        for t, b in enumerate(other):
            if (m >> t) & 1:
                base |= 1 << b
        rows: Dict[int, int] = {}                  # row index -> byte address of byte 0
        for l in range(32):
            h0 = base
            for t, b in enumerate(lane_bits):
                if (l >> t) & 1:
                    h0 |= 1 << b
            for e in range(1 << k):                # element e of the word (byte e·w)
                h = h0
                for t, b in enumerate(word_bits):
                    if (e >> t) & 1:
                        h |= 1 << b
                addr = int(S_inv[apply(L, h)]) * w
                if trans:
                    row, col_byte = 2 * (l % 4) + e, 2 * (l // 4)
                else:
                    row, col_byte = l // 4, 4 * (l % 4) + e * w
                start = addr - col_byte
                if start % 16 or rows.setdefault(row, start) != start:
                    raise ValueError("the instruction's tile does not divide M^-1∘L (Thm 5.1)")
        per_group: Dict[int, int] = {}
        for start in set(rows.values()):
            g = (start // group_bytes) % 8
            per_group[g] = per_group.get(g, 0) + 1
        total += max(per_group.values())
        ideal += 1
    return total, ideal


# --------------------------------------------------------------------------------------
# F2 helpers over sets of logical vectors (spans, completion) — used by the paper's
# shuffle and swizzle constructions
# --------------------------------------------------------------------------------------

def _reduce(v: int, basis: Dict[int, int]) -> int:
    while v:
        lead = v.bit_length() - 1
        if lead not in basis:
            return v
        v ^= basis[lead]
    return 0


def _echelon(vecs: Sequence[int]) -> Dict[int, int]:
    basis: Dict[int, int] = {}
    for v in vecs:
        r = _reduce(v, basis)
        if r:
            basis[r.bit_length() - 1] = r
    return basis


def in_span(v: int, vecs: Sequence[int]) -> bool:
    return _reduce(v, _echelon(vecs)) == 0


def rank(vecs: Sequence[int]) -> int:
    return len(_echelon(vecs))


def complete_basis(vecs: Sequence[int], d: int) -> List[int]:
    """Unit vectors (ascending flat order) completing span(vecs) to F2^d."""
    basis = _echelon(vecs)
    out = []
    for t in range(d):
        r = _reduce(1 << t, basis)
        if r:
            basis[r.bit_length() - 1] = r
            out.append(1 << t)
    return out


def span(vecs: Sequence[int]) -> set:
    s = {0}
    for v in vecs:
        s |= {x ^ v for x in s}
    return s


# --------------------------------------------------------------------------------------
# Intra-warp shuffle sets
# --------------------------------------------------------------------------------------

def shuffle_sets(A: Layout, B: Layout, w: int, max_bytes: int = 4):
    """The sets of P:375-387 for one warp: V (vectorisation, ≤ max_bytes per shuffle,
    candidates in A's register order, G9), I = A_Thr ∩ B_Thr, E = A_Thr \\ I,
    F = B_Thr \\ I (both ascending, G8), G = {e_i ⊕ f_i}, R completing V∪I∪G to the
    warp's space (unit vectors ascending).  Rounds = 2^|R|.  Assumes no broadcast
    (P:373).  Warp space = span of A's reg and lane columns."""
    a_reg, b_reg = A.cols_of("reg"), B.cols_of("reg")
    a_thr, b_thr = A.cols_of("lane"), B.cols_of("lane")
    V = []
    for c in a_reg:
        if c in b_reg and (1 << (len(V) + 1)) * w <= max_bytes:
            V.append(c)
    I = [c for c in a_thr if c in b_thr]
    E = sorted(c for c in a_thr if c not in I)
    F = sorted(c for c in b_thr if c not in I)
    assert len(E) == len(F), "broadcast is not handled by the basic algorithm (P:373)"
    G = [e ^ f for e, f in zip(E, F)]
    warp_space = a_reg + a_thr
    d_w = rank(warp_space)
    # R: complete V ∪ I ∪ G inside span(warp_space): take warp_space vectors in order
    basis = _echelon(V + I + G)
    R = []
    for c in sorted(warp_space):
        r = _reduce(c, basis)
        if r:
            basis[r.bit_length() - 1] = r
            R.append(c)
    assert len(V) + len(I) + len(G) + len(R) == d_w
    return dict(V=V, I=I, E=E, F=F, G=G, R=R, rounds=1 << len(R))


# --------------------------------------------------------------------------------------
# Optimal swizzling (P:391-426 main text; P:696-756 appendix)
# --------------------------------------------------------------------------------------

def optimal_swizzle(A: Layout, B: Layout, w: int, max_vec_bytes: int = 16,
                    segment_bytes: int = 128, bank_bytes: int = 4) -> Dict[str, List[int]]:
    """The paper's swizzle construction, step by step:

    1. V: basis of A_Reg ∩ B_Reg "as done for warp shuffles", ≤ max_vec_bytes (G9);
    2. b = log2(segment_bytes / (2^v·w))  (P:406, 128 on NVIDIA);
    3. A_Bank, B_Bank: A_Thr, B_Thr without their last log2 max(1, 2^v·w/4) vectors;
    4. E = A_Bank \\ B_Bank, F = B_Bank \\ A_Bank (|E| ≤ |F| after a swap), ordered
       ascending (G13); H = {e_i ⊕ f_i};
    5. C: completion of span(Vec ∪ A_Bank ∪ B_Bank) (unit vectors ascending);
    6. Seg: ℓ = d - v - b vectors from H then C; if too few, add unused A_Bank then
       A_Thr vectors (G14, P:424 / P:754);
    7. Bank: completion of span(Vec ∪ Seg) (unit vectors ascending).
    The space is the CTA's logical space spanned by A's reg, lane and warp columns.
    Returns the column lists; the smem layout S maps offset bits (Vec, Bank, Seg)."""
    a_reg, b_reg = A.cols_of("reg"), B.cols_of("reg")
    a_thr = [c for c in A.cols_of("lane") if c]
    b_thr = [c for c in B.cols_of("lane") if c]
    space = [c for c in A.cols_of("reg") + A.cols_of("lane") + A.cols_of("warp") if c]
    d = rank(space)
    V = []
    for c in a_reg:
        if c and c in b_reg and (1 << (len(V) + 1)) * w <= max_vec_bytes:
            V.append(c)
    v = len(V)
    vec_bytes = (1 << v) * w
    b = max(0, (segment_bytes // vec_bytes).bit_length() - 1)
    drop = max(1, vec_bytes // bank_bytes).bit_length() - 1
    a_bank = a_thr[:len(a_thr) - drop] if drop else list(a_thr)
    b_bank = b_thr[:len(b_thr) - drop] if drop else list(b_thr)
    E = sorted(c for c in a_bank if c not in b_bank)
    F = sorted(c for c in b_bank if c not in a_bank)
    if len(E) > len(F):
        E, F = F, E
    H = [e ^ f for e, f in zip(E, F)]
    C = []
    basis = _echelon(V + a_bank + b_bank)
    for c in sorted(space):                       # completion inside the CTA space
        r = _reduce(c, basis)
        if r:
            basis[r.bit_length() - 1] = r
            C.append(c)
    ell = d - v - b
    seg: List[int] = []
    for c in H + C:
        if len(seg) < ell and not in_span(c, V + seg):
            seg.append(c)
    for c in a_bank + a_thr:                      # conflicts unavoidable
        if len(seg) < ell and not in_span(c, V + seg):
            seg.append(c)
    basis = _echelon(V + seg)
    bank = []
    for c in sorted(space):
        r = _reduce(c, basis)
        if r:
            basis[r.bit_length() - 1] = r
            bank.append(c)
    assert len(V) + len(bank) + len(seg) == d
    return dict(Vec=V, Bank=bank, Seg=seg, H=H, C=C, v=v, b=b, ell=ell)


def smem_layout_from_swizzle(sw: Dict[str, List[int]], out_dims) -> Layout:
    """S: offset bits (Vec, Bank, Seg in that order) -> logical."""
    cols = list(sw["Vec"]) + list(sw["Bank"]) + list(sw["Seg"])
    return layout_from_cols([("offset", len(cols))], out_dims, cols)


def lemma95_optimum(U: Sequence[int], V: Sequence[int], d: int) -> int:
    """Lemma 9.5: the largest subspace with trivial intersection with
    U ∪ V has dimension d - max(dim U, dim V)."""
    return d - max(rank(U), rank(V))


# --------------------------------------------------------------------------------------
# O10  Gather along an axis (§5.5)
# --------------------------------------------------------------------------------------

def gather(L: Layout, axis: int, src: np.ndarray, idx: np.ndarray) -> np.ndarray:
    """src, idx and dst are packed in the same layout L.  In logical space,
    out[x] = src[x with the axis coordinate replaced by (axis(x) & ~(K-1)) |
    (idx[x] & (K-1))], K = 2^(number of non-block bits of L on the axis)
    (take_along_axis inside each tile; out-of-range indices masked, G16)."""
    nd = len(L.out_dims)
    shape = [1 << b for _, b in L.out_dims]
    axis_shift = sum(b for _, b in L.out_dims[axis + 1:])
    axis_mask = ((1 << L.out_dims[axis][1]) - 1) << axis_shift
    nonblock = [k for n, _ in L.in_dims if n != "block" and n != "dev"
                for k in L.dim_bits(n)]
    axis_bits = [L.cols[k] for k in nonblock if L.cols[k] & axis_mask]
    K = 1 << len(axis_bits)
    assert sorted(axis_bits) == [1 << (axis_shift + t) for t in range(len(axis_bits))], \
        "the in-tile axis bits must be the low bits of the axis coordinate"
    x_of_h = image_table(L).astype(np.int64)
    T_src = np.empty(int(np.prod(shape)), dtype=np.asarray(src).dtype)
    T_idx = np.empty(int(np.prod(shape)), dtype=np.int64)
    T_src[x_of_h] = np.asarray(src).reshape(-1)
    T_idx[x_of_h] = np.asarray(idx).reshape(-1)
    xs = np.arange(T_src.size, dtype=np.int64)
    a = (xs & axis_mask) >> axis_shift
    new_a = (a & ~(K - 1)) | (T_idx & (K - 1))
    src_x = (xs & ~axis_mask) | (new_a << axis_shift)
    T_out = T_src[src_x]
    return T_out[x_of_h]


# --------------------------------------------------------------------------------------
# O11  Reduction (sum) with broadcast de-duplication (Table 4)
# --------------------------------------------------------------------------------------

def reduce_ref_fp64(L: Layout, axis: int, src: np.ndarray, op: str = "sum") -> np.ndarray:
    """out[y] = Σ (op = "sum"; or max / min) over logical x whose non-(in-tile)-axis part
    is y of T[x], in fp64 (max / min are exact: the result is one of the fp32 inputs).
    The in-tile axis bits are the non-block axis bits of L; the output is the logical
    tensor with the axis replaced by its block part (row-major).  Table 4
    benchmarks `tl.sum`-style reductions; max and min are the other common ones."""
    shape = [1 << b for _, b in L.out_dims]
    x_of_h = image_table(L).astype(np.int64)
    T = np.empty(int(np.prod(shape)), dtype=np.float64)
    T[x_of_h] = np.asarray(src, dtype=np.float64).reshape(-1)
    axis_shift = sum(b for _, b in L.out_dims[axis + 1:])
    nonblock = [k for n, _ in L.in_dims if n not in ("block", "dev") for k in L.dim_bits(n)]
    axis_mask = ((1 << L.out_dims[axis][1]) - 1) << axis_shift
    kbits = len([k for k in nonblock if L.cols[k] & axis_mask])
    K = 1 << kbits
    new_shape = shape.copy()
    new_shape[axis] = shape[axis] // K
    T = T.reshape(shape[:axis] + [shape[axis] // K, K] + shape[axis + 1:])
    return {"sum": T.sum, "max": T.max, "min": T.min}[op](axis=axis + 1).reshape(-1)


def reduce_fixed_order_fp32(L: Layout, axis: int, src: np.ndarray) -> np.ndarray:
    """The fixed-order fp32 replica (the paper fixes no order, so the
    order is reading R-reduce), in LOGICAL coordinates: with the in-tile
    axis coordinate a in [0, K) (the low K bits of the axis, as for O10), for
    t = 0, 1, ..., log2 K - 1 in ascending order combine the pairs that differ only in
    bit t of a,  v <- v(t = 0) + v(t = 1)  (fp32, round to nearest, no FMA) — i.e. the
    recursive halving (pairwise) sum  S(x) = S(x[:K/2]) + S(x[K/2:]).  The result is a
    function of the logical tensor alone: it does not depend on how L places the bits
    on registers, lanes or warps, and broadcast (zero-column) copies of L
    contribute once.  Output: the logical tensor with the axis replaced by its block
    part, row-major (as reduce_ref_fp64)."""
    shape = [1 << b for _, b in L.out_dims]
    x_of_h = image_table(L).astype(np.int64)
    T = np.empty(int(np.prod(shape)), dtype=np.float32)
    T[x_of_h] = np.asarray(src, dtype=np.float32).reshape(-1)
    axis_shift = sum(b for _, b in L.out_dims[axis + 1:])
    axis_mask = ((1 << L.out_dims[axis][1]) - 1) << axis_shift
    nonblock = [k for n, _ in L.in_dims if n not in ("block", "dev") for k in L.dim_bits(n)]
    kbits = len([k for k in nonblock if L.cols[k] & axis_mask])
    K = 1 << kbits
    # [outer, tiles along the axis, K, inner]: the in-tile axis coordinate is axis 2
    v = T.reshape(int(np.prod(shape[:axis], dtype=np.int64)), shape[axis] // K, K,
                  int(np.prod(shape[axis + 1:], dtype=np.int64)))
    for t in range(kbits):
        # after t steps, position q of axis 2 holds the sum over the aligned block of
        # 2^t original positions q*2^t ...; bit t of a is now the lowest bit of q
        v = (v[:, :, 0::2, :] + v[:, :, 1::2, :]).astype(np.float32)
    return v.reshape(-1)


# --------------------------------------------------------------------------------------
# O13  Scan (inclusive prefix sum) along an axis inside each tile ("reduction and
#      scan operations").  The paper fixes no scan algorithm; reading
#      R-scan: the in-tile axis is the low K bits of the axis coordinate
#      (as for gather / reduce), and the fp32 order is the bit-doubling recurrence below,
#      written in logical coordinates so that it does not depend on any hardware mapping.
# --------------------------------------------------------------------------------------

def _scan_setup(L: Layout, axis: int, src: np.ndarray, dtype):
    shape = [1 << b for _, b in L.out_dims]
    x_of_h = image_table(L).astype(np.int64)
    T = np.empty(int(np.prod(shape)), dtype=dtype)
    T[x_of_h] = np.asarray(src, dtype=dtype).reshape(-1)
    axis_shift = sum(b for _, b in L.out_dims[axis + 1:])
    axis_mask = ((1 << L.out_dims[axis][1]) - 1) << axis_shift
    nonblock = [k for n, _ in L.in_dims if n not in ("block", "dev") for k in L.dim_bits(n)]
    kbits = len([k for k in nonblock if L.cols[k] & axis_mask])
    T = T.reshape(shape[:axis] + [shape[axis] >> kbits, 1 << kbits] + shape[axis + 1:])
    return T, kbits, x_of_h, shape


def scan_ref_fp64(L: Layout, axis: int, src: np.ndarray, op: str = "sum") -> np.ndarray:
    """out[x] = sum (op = "sum"; or max / min) of T[x with axis coordinate a'] over the a'
    of x's tile with a' <= a(x) (inclusive), in fp64, returned packed in L like the input
    (library cumsum / running maximum / running minimum; max and min are exact)."""
    T, kbits, x_of_h, shape = _scan_setup(L, axis, src, np.float64)
    acc = {"sum": np.cumsum, "max": np.maximum.accumulate, "min": np.minimum.accumulate}[op]
    out = acc(T, axis=axis + 1).reshape(-1)
    return out[x_of_h]


def scan_bitdoubling_fp32(L: Layout, axis: int, src: np.ndarray) -> np.ndarray:
    """The fixed-order fp32 scan (reading R-scan), in logical coordinates, step by step:
    for t = 0 .. K_bits-1, every element whose in-tile axis coordinate a has bit t set
    adds the value, before this step, of the last element of the lower half of its
    aligned 2^(t+1)-block, a' = (a with bit t cleared) | (2^t - 1):
        v[a] <- v[a] + v[a']   (fp32, round to nearest; simultaneous update).
    After step t every element holds the inclusive sum of its aligned 2^(t+1)-block
    prefix; after the last step, the in-tile inclusive prefix sum."""
    T, kbits, x_of_h, shape = _scan_setup(L, axis, src, np.float32)
    ax = axis + 1
    K = 1 << kbits
    v = T.copy()
    a = np.arange(K)
    for t in range(kbits):
        upper = (a >> t) & 1 == 1
        partner = (a & ~((2 << t) - 1)) | ((1 << t) - 1)
        src_vals = np.take(v, partner[upper], axis=ax)
        cur = np.take(v, a[upper], axis=ax)
        new = (cur + src_vals).astype(np.float32)
        idx = [slice(None)] * v.ndim
        idx[ax] = a[upper]
        v[tuple(idx)] = new
    return v.reshape(-1)[x_of_h]


# --------------------------------------------------------------------------------------
# O12  Distributed view (dev input dimension declared last)
# --------------------------------------------------------------------------------------

def rank_slice(L: Layout, r: int) -> Layout:
    """The local layout of rank r: L with the dev bits fixed to r, as an affine map;
    returned as (local layout, offset flat) — the local layout drops the dev dim."""
    in_local = [(n, b) for n, b in L.in_dims if n != "dev"]
    bases = {n: L.bases[n] for n, _ in in_local}
    loc = Layout(in_local, list(L.out_dims), bases)
    dev_bits = L.dim_bits("dev")
    off = 0
    for t, k in enumerate(dev_bits):
        if (r >> t) & 1:
            off ^= L.cols[k]
    return loc, off


def convert_distributed_rank(A: Layout, B: Layout, T: np.ndarray, r: int) -> np.ndarray:
    """Rank r's slice of convert(A, B) computed from the logical tensor T:
    dst_r[h] = T[B(h, dev=r)] (closed form of O5 with dev as the top input bits)."""
    locB, offB = rank_slice(B, r)
    xs = apply_all(locB, np.arange(1 << locB.d_in, dtype=np.uint64)) ^ np.uint64(offB)
    return np.asarray(T).reshape(-1)[xs.astype(np.int64)]


def enumerate_bijective_relabelings(d: int):
    """All d! assignments of d logical unit vectors to d hardware bits (E1)."""
    return itertools.permutations([1 << t for t in range(d)])
