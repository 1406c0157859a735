"""Pins for the CPU oracle (oracle/ll_oracle.py) against what the paper and the
mathematics fix — NOT against the oracle itself.  Each test names its pin.
All run on CPU (-m "not gpu")."""
import itertools
import json
import os

import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def L_of(spec):
    return O.Layout(*W.spec_to_bases(spec))


# ----------------------------------------------------------------------------- GV1/GV2

def fig1_A_from_matrix():
    g = load("fig1_table1.json")
    rows = g["matrix_A_rows"]
    out_dims = [tuple(d) for d in g["out_dims"]]
    names = ["reg", "reg", "lane", "lane", "lane", "lane", "lane", "warp"]
    bases = {"reg": [], "lane": [], "warp": []}
    for col in range(8):
        i = sum(rows[f"i{k}"][col] << k for k in range(4))
        j = sum(rows[f"j{k}"][col] << k for k in range(4))
        bases[names[col]].append((i, j))
    return O.Layout([tuple(d) for d in g["in_dims"]], out_dims, bases), g


def test_table1_rows_reproduced_by_matrix_A():
    """GV1: every printed row of Table 1 equals A·v with the P:140 matrix,
    and the min-index preimage maps it back (A is bijective)."""
    A, g = fig1_A_from_matrix()
    first = O.preimage_min(A)
    for i, j, r, t, w in g["table1_ij_reg_thread_warp"]:
        h = O.hw_flat(A.in_dims, (r, t, w))
        assert O.logical_coords(A.out_dims, O.apply(A, h)) == (i, j)
        assert first[O.logical_flat(A.out_dims, (i, j))] == h
    assert O.is_injective(A) and O.is_surjective(A)


def test_worked_example_r1_t9_w0():
    """GV2: loc_r1=(0,1), loc_t9=(2,2), loc_w0=(0,0), XOR=(2,3)."""
    A, g = fig1_A_from_matrix()
    ex = g["worked_example"]
    loc = lambda r, t, w: O.logical_coords(A.out_dims, O.apply(A, O.hw_flat(A.in_dims, (r, t, w))))
    assert loc(ex["reg"], 0, 0) == tuple(ex["loc_reg"])
    assert loc(0, ex["thread"], 0) == tuple(ex["loc_thread"])
    assert loc(0, 0, ex["warp"]) == tuple(ex["loc_warp"])
    assert loc(ex["reg"], ex["thread"], ex["warp"]) == tuple(ex["ij"])


def test_blocked_constructor_is_fig1_A():
    """GV3 (P:128 vs P:140): blocked([2,2],[4,8],[2,1],[1,0]) on 16x16 == matrix A."""
    A, g = fig1_A_from_matrix()
    p = g["blocked_params_P128"]
    Lb = O.blocked(p["shape"], p["size_per_thread"], p["threads_per_warp"], p["warps_per_cta"], p["order"])
    assert Lb.cols == A.cols


def test_fig1_literal_tables_match_matrix():
    A, _ = fig1_A_from_matrix()
    assert L_of(W.C1_A).cols == A.cols


@pytest.mark.parametrize("which,ctor", [
    ("c2B", lambda: O.blocked([128, 128], [8, 8], [2, 16], [4, 1], [1, 0])),
    ("c3A", lambda: O.blocked([256, 128], [1, 8], [2, 16], [4, 1], [1, 0])),
    ("c3B", lambda: O.blocked([256, 128], [8, 1], [32, 1], [1, 4], [0, 1])),
    ("c3bA", lambda: O.blocked([256, 128], [8, 8], [2, 16], [4, 1], [1, 0])),
    ("c3bB", lambda: O.blocked([256, 128], [8, 8], [32, 1], [1, 4], [0, 1])),
    ("c2A", lambda: O.mma_acc([128, 128], 4)),
])
def test_constructors_match_appendix_tables(which, ctor):
    tbl = {"c2B": W.c2(0)[1], "c3A": W.c3(0)[0], "c3B": W.c3(0)[1],
           "c3bA": W.c3b(0)[0], "c3bB": W.c3b(0)[1], "c2A": W.c2(0)[0]}[which]
    lit = L_of(tbl)
    got = ctor()
    # compare per hardware bit, on the tile dims (drop the empty batch dim)
    assert [c for c in got.cols] == [c for c in lit.cols]


def test_mma_acc_matches_ptx_fragment():
    """Prop 9.2 vs the PTX m16n8 C/D fragment [HW]: element d[k] of lane l
    sits at row = l/4 + 8*(k/2 % 2), col = 2*(l % 4) + k % 2, repeated over n in
    8-column blocks then over m in 16-row blocks (wgmma: warps along M, 16 rows)."""
    L = O.mma_acc([128, 128], 4)
    ntile = 128 // 8
    for h in range(1 << L.d_in):
        r = h & 127
        lane = (h >> 7) & 31
        warp = h >> 12
        q = r & 3                 # position in the m16n8 fragment
        nrep = (r >> 2) & (ntile - 1)
        mrep = r >> (2 + 4)
        row = lane // 4 + 8 * (q // 2) + 16 * warp + 64 * mrep
        col = 2 * (lane % 4) + q % 2 + 8 * nrep
        # the register numbering of Prop 9.2 is reg0 -> j0, reg1 -> i3 (G17)
        assert O.logical_coords(L.out_dims, O.apply(L, h)) == (row, col)


# ----------------------------------------------------------------------------- GV4

def test_mma_swizzle_linear_and_C_rows():
    """GV4: the [[I_n, C],[0, I_m]] layout equals the Def 4.11 formula at all
    4096 points, and its C rows equal the P:264 values."""
    g = load("mma_swizzle_C.json")
    m, n = g["m"], g["n"]
    for case in g["cases"]:
        vec, pp, mp = case["vec"], case["per_phase"], case["max_phase"]
        assert O.mma_swizzle_C(m, n, vec, pp, mp) == case["C"]
        L = O.mma_swizzle_layout(m, n, vec, pp, mp)
        for i in range(1 << m):
            for j in range(1 << n):
                off = O.apply(L, j | (i << n))
                assert off == (i << n) + O.mma_swizzle_offset(i, j, vec, pp, mp)
        assert O.is_memory(L)


# ----------------------------------------------------------------------------- predicates

@pytest.mark.parametrize("ctor", [
    lambda: O.blocked([16, 16], [2, 2], [4, 8], [2, 1], [1, 0]),
    lambda: O.blocked([8, 8], [1, 1], [4, 8], [2, 1], [1, 0]),     # broadcast: 64 < 256 slots
    lambda: O.mma_acc([64, 32], 4),
    lambda: O.mma_acc([16, 8], 1),
])
def test_blocked_and_mma_are_distributed(ctor):
    """P:206 (blocked), P:212 (mma) with Def 4.10."""
    assert O.is_distributed(ctor())


def test_sliced_is_surjective_maybe_not_injective():
    """Remark P:224: a slice stays surjective, may lose injectivity."""
    L = O.blocked([16, 16], [2, 2], [4, 8], [2, 1], [1, 0])
    S = O.sliced(L, 1)
    assert O.is_surjective(S) and not O.is_injective(S)
    zero = [c for c in S.cols if c == 0]
    assert len(zero) == 4          # the j bits became zero (broadcast) columns


# ----------------------------------------------------------------------------- inverse

def test_right_inverse_equals_min_index_preimage_random():
    """Slack-zero Gaussian elimination == brute-force min-index
    preimage, and A∘A^+ = I (Def 4.5)."""
    rng = np.random.default_rng(7)
    for trial in range(600):
        d_out = int(rng.integers(1, 7))
        d_in = int(rng.integers(d_out, 10))
        cols = gen.random_surjective_cols(rng, d_out, d_in)
        L = O.layout_from_cols([("h", d_in)], [("x", d_out)], cols)
        first = O.preimage_min(L)
        xs = np.arange(1 << d_out, dtype=np.uint64)
        assert np.array_equal(O.apply_inverse_all(L, xs).astype(np.int64), first)
        assert np.array_equal(O.apply_all(L, first.astype(np.uint64)), xs)


def test_inverse_of_injective_is_two_sided():
    rng = np.random.default_rng(11)
    for _ in range(50):
        d = int(rng.integers(1, 9))
        cols = gen.random_memory_cols(rng, d)
        L = O.layout_from_cols([("offset", d)], [("x", d)], cols)
        Li = O.right_inverse(L)
        hs = np.arange(1 << d, dtype=np.uint64)
        assert np.array_equal(O.apply_all(Li, O.apply_all(L, hs)), hs)     # A^+∘A = I
        assert O.is_memory(L)


def test_left_inverse_fails_for_broadcast():
    """A^+∘A = I iff A is injective (zero columns are lost)."""
    L = O.blocked([8, 8], [1, 1], [4, 8], [2, 1], [1, 0])
    Li = O.right_inverse(L)
    hs = np.arange(1 << L.d_in, dtype=np.uint64)
    assert not np.array_equal(O.apply_all(Li, O.apply_all(L, hs)), hs)


def test_nonsurjective_has_no_right_inverse():
    L = O.layout_from_cols([("h", 3)], [("x", 3)], [1, 2, 3])
    with pytest.raises(ValueError):
        O.right_inverse(L)
    with pytest.raises(ValueError):
        O.preimage_min(L)


# ----------------------------------------------------------------------------- compose etc.

def test_compose_is_function_composition_and_associative():
    """Def 4.2: (L2∘L1)(u) = L2(L1(u)); associativity."""
    rng = np.random.default_rng(3)
    for _ in range(40):
        a, b, c, d = (int(x) for x in rng.integers(1, 7, size=4))
        L1 = O.layout_from_cols([("u", a)], [("v", b)], [int(x) for x in rng.integers(0, 1 << b, a)])
        L2 = O.layout_from_cols([("v", b)], [("w", c)], [int(x) for x in rng.integers(0, 1 << c, b)])
        L3 = O.layout_from_cols([("w", c)], [("z", d)], [int(x) for x in rng.integers(0, 1 << d, c)])
        C = O.compose(L2, L1)
        for u in range(1 << a):
            assert O.apply(C, u) == O.apply(L2, O.apply(L1, u))
        assert O.compose(L3, C).cols == O.compose(O.compose(L3, L2), L1).cols


def test_product_then_left_division_roundtrip():
    """(M1 × M2) /_l M1 = M2 (Defs 4.3, 4.4)."""
    M1 = O.blocked([4, 4], [2, 2], [2, 2], [1, 1], [1, 0])
    M2 = O.blocked([8, 4], [1, 2], [4, 2], [2, 1], [1, 0])
    M1 = O.Layout(M1.in_dims, [("d0", 2), ("d1", 2)], M1.bases)
    P = O.product(M1, M2)
    Q = O.left_divide(P, M1)
    assert Q.cols == M2.cols
    # block-diagonal structure: M1 bits stay inside M1's range
    with pytest.raises(ValueError):
        O.left_divide(P, M2)


def test_left_divide_ldst_tile():
    """Thm 5.1 with the vectorised ld/st tile: a layout whose two lowest
    register bits are the two lowest offset bits is divisible by id_2^{Reg,Off}."""
    T = O.Layout([("reg", 2)], [("offset", 2)], {"reg": [(1,), (2,)]})
    L = O.Layout([("reg", 3), ("lane", 1)], [("offset", 4)], {"reg": [(1,), (2,), (8,)], "lane": [(4,)]})
    R = O.left_divide(L, T)
    assert R.cols == [2, 1]
    L_bad = O.Layout([("reg", 3), ("lane", 1)], [("offset", 4)], {"reg": [(2,), (1,), (8,)], "lane": [(4,)]})
    with pytest.raises(ValueError):
        O.left_divide(L_bad, T)


# ----------------------------------------------------------------------------- convert

def test_convert_closed_form_pack():
    """O5: convert(pack_A(T)) == pack_B(T) for Fig. 1 A -> B and the batch variant."""
    rng = np.random.default_rng(1001)
    A, B = L_of(W.C1_A), L_of(W.C1_B)
    T = gen.random_bits(rng, 256, 4)
    assert np.array_equal(O.convert(A, B, O.pack(A, T)), O.pack(B, T))
    A2, B2 = (L_of(s) for s in W.c1_batched(3))
    T2 = gen.random_bits(rng, 256 * 8, 4)
    assert np.array_equal(O.convert(A2, B2, O.pack(A2, T2)), O.pack(B2, T2))


def test_convert_identity_and_transpose_library():
    """A = B is the identity; row-major -> column-major memory layouts is
    numpy.transpose (a library routine)."""
    rng = np.random.default_rng(5)
    out = [("i", 3), ("j", 4)]
    row = O.identity_memory(out)
    col = O.layout_from_cols([("offset", 7)], out, [1 << (4 + k) for k in range(3)] + [1 << k for k in range(4)])
    T = gen.random_bits(rng, 128, 2)
    assert np.array_equal(O.convert(row, row, T), T)
    got = O.convert(row, col, T)
    assert np.array_equal(got, T.reshape(8, 16).T.reshape(-1))


def test_convert_random_exhaustive_small():
    """Exhaustive 2^8 spaces (E1 subsample): random bijective B against Fig. 1 A;
    closed form and A-consistency; broadcast variant with zero columns."""
    rng = np.random.default_rng(2024)
    A = L_of(W.C1_A)
    hw = [("reg", 2), ("lane", 5), ("warp", 1)]
    T = gen.random_bits(rng, 256, 4)
    for _ in range(200):
        B = L_of(gen.random_distributed(rng, W.C1_OUT, hw))
        assert np.array_equal(O.convert(A, B, O.pack(A, T)), O.pack(B, T))
    out7 = [("i", 3), ("j", 4)]
    T7 = gen.random_bits(rng, 128, 4)
    for _ in range(200):
        A7 = L_of(gen.random_distributed(rng, out7, hw, zero_ok=["reg"]))
        B7 = L_of(gen.random_distributed(rng, out7, hw, zero_ok=["lane"]))
        src = O.pack(A7, T7)
        assert O.is_consistent(A7, src)
        assert np.array_equal(O.convert(A7, B7, src), O.pack(B7, T7))


def test_convert_at_matches_full_convert():
    rng = np.random.default_rng(9)
    A, B = (L_of(s) for s in W.c1_batched(4))
    T = gen.random_bits(rng, 256 * 16, 4)
    src = O.pack(A, T)
    full = O.convert(A, B, src)
    hs = rng.integers(0, 1 << B.d_in, size=500).astype(np.uint64)
    assert np.array_equal(O.convert_at(A, B, src, hs), full[hs.astype(np.int64)])


# ----------------------------------------------------------------------------- class

def test_class_special_cases():
    """O7 on cases the paper fixes: A = B is NOOP; swapping A's register bits is a
    register permutation; Fig.1 A->B^T needs smem (warp bit moves)."""
    A = L_of(W.C1_A)
    assert O.classify(A, A) == "NOOP"
    swapped = {"out": W.C1_OUT, "in": [("reg", ["i0", "j0"]), ("lane", ["j1", "j2", "j3", "i1", "i2"]), ("warp", ["i3"])]}
    assert O.classify(A, L_of(swapped)) == "REGPERM"
    lane_perm = {"out": W.C1_OUT, "in": [("reg", ["j0", "i0"]), ("lane", ["j2", "j1", "j3", "i1", "i2"]), ("warp", ["i3"])]}
    assert O.classify(A, L_of(lane_perm)) == "SHUFFLE"
    assert O.classify(A, L_of(W.C1_B)) == "SMEM"
    A2, B2 = (L_of(s) for s in W.c1_batched(2))
    blk = {"out": A2.out_dims, "in": [("reg", ["j0", "i0"]), ("lane", ["j1", "j2", "j3", "i1", "i2"]),
                                       ("warp", ["b0"]), ("block", ["i3", "b1"])]}
    assert O.classify(A2, L_of(blk)) == "CTA"


def test_class_configs_2_3():
    A, B = (L_of(s) for s in W.c2(0))
    assert O.classify(A, B) == "SHUFFLE"
    A, B = (L_of(s) for s in W.c3(0))
    assert O.classify(A, B) == "SMEM"


def test_class_config5_device():
    for p in (1, 2):
        A, B = (L_of(s) for s in W.c5(p, n=4))
        assert O.classify(A, B) == "DEVICE"


def test_class_config5_p0_noop_and_transpose_cta():
    A, B = (L_of(s) for s in W.c5(0, n=4))
    assert O.classify(A, B) == "NOOP"
    A, B = (L_of(s) for s in W.c5T(0, n=3))
    assert O.classify(A, B) == "CTA"


# ----------------------------------------------------------------------------- shuffle

def test_shuffle_cosets_hold_one_vector_per_lane():
    """for each i, R(i) ⊕ span(V∪I∪G) contains exactly one vectorised element
    per thread of A and of B; the rounds cover every register once.  Checked
    exhaustively (all 2^|R| cosets) on random SHUFFLE-class pairs."""
    rng = np.random.default_rng(42)
    out = [("i", 4), ("j", 4)]
    hw = [("reg", 3), ("lane", 5)]
    tested = 0
    for _ in range(400):
        A = L_of(gen.random_distributed(rng, out, hw))
        B = L_of(gen.random_distributed(rng, out, hw))
        if O.classify(A, B) != "SHUFFLE":
            continue
        for w in (1, 2, 4):
            s = O.shuffle_sets(A, B, w)
            assert s["rounds"] == 1 << ((3 + 5) - len(s["V"]) - len(s["I"]) - len(s["G"]))
            base = O.span(s["V"] + s["I"] + s["G"])
            vecspan = O.span(s["V"])
            Ainv, Binv = O.preimage_min(A), O.preimage_min(B)
            seen_a = set()
            for ri in range(s["rounds"]):
                r = 0
                for t, c in enumerate(s["R"]):
                    if (ri >> t) & 1:
                        r ^= c
                coset = {r ^ x for x in base}
                for L, inv, seen in ((A, Ainv, seen_a), (B, Binv, None)):
                    lanes = {}
                    for x in coset:
                        h = int(inv[x])
                        lane = (h >> 3) & 31
                        lanes.setdefault(lane, set()).add(x)
                    assert sorted(lanes) == list(range(32))
                    for lane, xs in lanes.items():
                        x0 = min(xs)
                        assert xs == {x0 ^ v for v in vecspan}   # one vector per lane
                        if seen is not None:
                            seen.add(x0)
            assert len(seen_a) * len(vecspan) == 256
        tested += 1
    assert tested >= 20


# ----------------------------------------------------------------------------- swizzle

def _fig5():
    g = load("fig5_swizzle.json")
    out = [tuple(d) for d in g["out_dims"]]
    A = L_of({"out": out, "in": [(k, v) for k, v in g["A"].items()]})
    B = L_of({"out": out, "in": [(k, v) for k, v in g["B"].items()]})
    return A, B, g


def test_fig5_swizzle_reproduces_P426_schedule():
    """GV5 (P:426 under the G3 reconstruction): Vec=[r0], Bank=[c0], Seg=[c0^c1, r1];
    the read schedule printed in the paper; no conflicts in reads or writes."""
    A, B, g = _fig5()
    sw = O.optimal_swizzle(A, B, g["elem_bytes"], segment_bytes=g["segment_bytes"],
                           bank_bytes=g["bank_bytes"])
    flat = lambda name: O.logical_flat(A.out_dims, W.bit_coords(A.out_dims, name))
    assert sw["Vec"] == [flat("r0")]
    assert sw["Bank"] == [flat("c0")]
    assert sw["Seg"] == [flat("c0") ^ flat("c1"), flat("r1")]
    S = O.smem_layout_from_swizzle(sw, A.out_dims)
    off = O.preimage_min(S)
    nbank = g["segment_bytes"] // g["bank_bytes"]
    for rd in g["reads_P426"]:
        t = rd["thread"]
        # element ids of the paper: id = 4r + c
        elems = []
        for r0 in (0, 1):
            h = r0 | (t << 2)
            x = O.apply(A, h)
            r, c = O.logical_coords(A.out_dims, x)
            elems.append(4 * r + c)
            assert int(off[x]) % nbank == rd["banks"][r0]
            assert int(off[x]) // nbank == rd["transaction"]  # segment index
        assert elems == rd["elements"]
    for L in (A, B):
        wf, ideal = O.smem_wavefronts(S, L, g["elem_bytes"], sw["Vec"], bank_bytes=g["bank_bytes"],
                                      n_banks=nbank)
        assert wf == ideal == 4      # "four transactions without bank conflicts"


@pytest.mark.parametrize("cfg", ["c1", "c3", "c3b"])
def test_swizzle_conflict_free_on_configs(cfg):
    """Lemma 9.4: the constructed S gives the ideal wavefront count for
    both the store (A) and the load (B) of configs 1, 3 and 3b."""
    A, B = {"c1": lambda: (L_of(W.C1_A), L_of(W.C1_B)),
            "c3": lambda: tuple(L_of(s) for s in W.c3(0)),
            "c3b": lambda: tuple(L_of(s) for s in W.c3b(0))}[cfg]()
    w = {"c1": 4, "c3": 2, "c3b": 2}[cfg]
    sw = O.optimal_swizzle(A, B, w)
    S = O.smem_layout_from_swizzle(sw, A.out_dims)
    assert O.is_memory(S) or all(bin(c).count("1") <= 2 for c in S.cols)
    for L in (A, B):
        wf, ideal = O.smem_wavefronts(S, L, w, sw["Vec"])
        assert wf == ideal


def test_unswizzled_config3_conflicts():
    """Sanity of the bank model: a row-major (unswizzled) buffer for config 3 is
    conflicted on the column-order side (4-way st / 32-way ld)."""
    A, B = (L_of(s) for s in W.c3(0))
    row = O.identity_memory(A.out_dims)
    # 1-element (2-byte) accesses
    wfA, idA = O.smem_wavefronts(row, A, 2, [])
    wfB, idB = O.smem_wavefronts(row, B, 2, [])
    assert wfA == 4 * idA      # 16 lanes at 16 B stride + the i0 lane: 4-way
    assert wfB == 32 * idB     # lanes run along i (256 B apart): all in one bank


def _mat_layouts(rows_log2_cols=3, trans=False):
    """One 8x8 b16 matrix held as the ldmatrix fragment (PTX m8n8 [HW]):
    non-transposed, reg bit -> j0, lanes 0,1 -> j1,j2, lanes 2-4 -> i0..i2; transposed,
    reg bit -> i0, lanes 0,1 -> i1,i2, lanes 2-4 -> j0..j2.  The smem buffer S is the
    row-major [8, 2^c] tensor (identity memory layout)."""
    out = [("i", 3), ("j", rows_log2_cols)]
    if trans:
        bases = {"reg": [(1, 0)], "lane": [(2, 0), (4, 0), (0, 1), (0, 2), (0, 4)]}
    else:
        bases = {"reg": [(0, 1)], "lane": [(0, 2), (0, 4), (1, 0), (2, 0), (4, 0)]}
    L = O.Layout([("reg", 1), ("lane", 5)], out, bases)
    return L, O.identity_memory(out)


def test_matrix_model_closed_forms():
    """Bank model of ldmatrix/stmatrix, pinned to textbook bank arithmetic
    (bank = byte address / 4 mod 32): an 8x8 b16 matrix stored densely (rows 16 B
    apart) covers one 128-byte segment — 1 wavefront; the same fragment in an [8, 64]
    b16 row-major tensor has its 8 rows 128 B apart, all in banks 0-3 — 8 wavefronts
    (8-way conflict); rows 32 B apart ([8, 16]) — 4 rows per group pair: 2-way."""
    for c, want in [(3, 1), (6, 8), (4, 2)]:
        L, S = _mat_layouts(c)
        # widen L with zero-free extra columns: the remaining j bits of the row as regs
        extra = [(0, 8 << t) for t in range(c - 3)]
        L = O.Layout([("reg", 1 + len(extra)), ("lane", 5)], L.out_dims,
                     {"reg": [(0, 1)] + extra, "lane": L.bases["lane"]})
        wf, ideal = O.smem_matrix_wavefronts(S, L, 2, [1])
        assert ideal == 1 << len(extra)
        assert wf == want * ideal, (c, wf, ideal)
    L, S = _mat_layouts(3, trans=True)
    assert O.smem_matrix_wavefronts(S, L, 2, [8], trans=True) == (1, 1)   # word: i0
    # the non-transposed fragment read with .trans is not a valid access
    L, S = _mat_layouts(3)
    with pytest.raises(ValueError):
        O.smem_matrix_wavefronts(S, L, 2, [1], trans=True)


def test_matrix_model_agrees_with_thm51_left_division():
    """Thm 5.1: the instruction lowers M^{-1}∘L iff M^{-1}∘L /_l T exists for
    T = id_k^{Reg,Off} × id_2^{Thr,Off}, k = log2(4/w).  Two independent
    formulations — the PTX fragment semantics of the bank model (raises when the
    rows are not 16 contiguous bytes) and the paper's left division (Def 4.4) — must
    agree on random bijective (reg, lane) -> smem-offset maps."""
    rng = np.random.default_rng(51)
    agree = {True: 0, False: 0}
    for w in (1, 2, 4):
        k = (4 // w).bit_length() - 1
        nreg = k + 2
        d = nreg + 5
        out = [("x", d)]
        T = O.Layout([("reg", k), ("lane", 2)], [("x", k + 2)],
                     {"reg": [(1 << i,) for i in range(k)], "lane": [(1 << (k + t),) for t in range(2)]})
        for case in range(150):
            perm = list(rng.permutation(d))
            if case % 3 == 0:                      # force the tile bits into place
                rest = [p for p in perm if p >= k + 2]
                pos = list(range(k)) + [nreg, nreg + 1]
                perm = [None] * d
                for b, p in zip(pos, range(k + 2)):
                    perm[b] = p
                it = iter(rest)
                perm = [p if p is not None else next(it) for p in perm]
            cols = [1 << int(p) for p in perm]
            L = O.layout_from_cols([("reg", nreg), ("lane", 5)], out, cols)
            S = O.identity_memory(out)
            try:
                O.smem_matrix_wavefronts(S, L, w, cols[:k])
                ok_model = True
            except ValueError:
                ok_model = False
            try:
                O.left_divide(L, T)
                ok_div = True
            except ValueError:
                ok_div = False
            assert ok_model == ok_div, (w, perm)
            agree[ok_div] += 1
    assert agree[True] >= 50 and agree[False] >= 50


def _all_subspaces(d, k):
    """All k-dim subspaces of F2^d as sorted tuples of their reduced bases."""
    seen = set()
    for combo in itertools.combinations(range(1, 1 << d), k):
        if O.rank(list(combo)) == k:
            key = tuple(sorted(O.span(list(combo))))
            if key not in seen:
                seen.add(key)
                yield list(combo)


def test_lemma95_bruteforce():
    """Lemma 9.5: largest subspace with trivial intersection with U ∪ V has dim
    d - max(dim U, dim V); brute force over all subspaces of F2^4."""
    rng = np.random.default_rng(0)
    d = 4
    for _ in range(25):
        U = [int(x) for x in rng.integers(1, 1 << d, size=int(rng.integers(1, 3)))]
        V = [int(x) for x in rng.integers(1, 1 << d, size=int(rng.integers(1, 3)))]
        su, sv = O.span(U), O.span(V)
        best = 0
        for k in range(d, 0, -1):
            if any(not ((O.span(b) - {0}) & (su | sv)) for b in _all_subspaces(d, k)):
                best = k
                break
        assert best == O.lemma95_optimum(U, V, d)


def test_swizzle_optimal_exhaustive_toy():
    """E2 (Lemmas 9.4-9.6): with a toy bank geometry (4 banks of 4 B per segment) and
    4 lanes, whenever some Seg subspace is conflict-free for both A and B, the
    paper's construction is conflict-free too; and it is conflict-free exactly when
    ℓ ≤ d - max(dim U, dim V) with U, V the Vec+Bank-lane spans (Lemma 9.5)."""
    rng = np.random.default_rng(77)
    out = [("r", 3), ("c", 2)]
    hw = [("reg", 3), ("lane", 2)]
    checked = 0
    for _ in range(60):
        A = L_of(gen.random_distributed(rng, out, hw))
        B = L_of(gen.random_distributed(rng, out, hw))
        w = 4
        sw = O.optimal_swizzle(A, B, w, segment_bytes=16, bank_bytes=4)
        if not sw["Vec"]:
            continue
        S = O.smem_layout_from_swizzle(sw, A.out_dims)
        tot = sum(O.smem_wavefronts(S, L, w, sw["Vec"], n_banks=4)[0] for L in (A, B))
        ideal = sum(O.smem_wavefronts(S, L, w, sw["Vec"], n_banks=4)[1] for L in (A, B))
        # brute force over all Seg subspaces complementing Vec
        d = 5
        best = None
        for seg in _all_subspaces(d, sw["ell"]) if sw["ell"] > 0 else [[]]:
            if O.rank(sw["Vec"] + seg) != len(sw["Vec"]) + len(seg):
                continue
            bank = O.complete_basis(sw["Vec"] + seg, d)
            S2 = O.smem_layout_from_swizzle({"Vec": sw["Vec"], "Bank": bank, "Seg": seg}, A.out_dims)
            t2 = sum(O.smem_wavefronts(S2, L, w, sw["Vec"], n_banks=4)[0] for L in (A, B))
            best = t2 if best is None else min(best, t2)
        if best == ideal:
            assert tot == ideal
        checked += 1
    assert checked >= 20


# ----------------------------------------------------------------------------- gather / reduce

@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_gather_is_take_along_axis(family):
    """O10 vs numpy.take_along_axis on the tile-reshaped tensor."""
    rng = np.random.default_rng(1004)
    L = L_of(W.c4("gather", family, n_i=8, n_j=7))     # [256, 128] with [128, 32] tiles
    n = 1 << L.d_in
    T = gen.random_bits(rng, n, 4)
    Ti = rng.integers(0, 32, size=n).astype(np.int32)
    out = O.gather(L, 1, O.pack(L, T), O.pack(L, Ti))
    ref = np.take_along_axis(T.reshape(256, 4, 32), Ti.reshape(256, 4, 32).astype(np.int64), axis=2)
    assert np.array_equal(out, O.pack(L, ref.reshape(-1)))


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_reduce_fp64_and_fixed_order(family):
    """O11: fp64 reference equals numpy's sum over [128,128] tiles; the fixed-order
    fp32 replica is within 1e-6 relative (U[0,1) inputs, no cancellation)."""
    rng = np.random.default_rng(1005)
    L = L_of(W.c4("reduce", family, n_i=8, n_j=8))     # [256, 256] with [128,128] tiles
    n = 1 << L.d_in
    T = rng.random(n, dtype=np.float32)
    src = O.pack(L, T)
    ref = O.reduce_ref_fp64(L, 1, src)
    lib = T.astype(np.float64).reshape(256, 2, 128).sum(axis=2).reshape(-1)
    assert np.allclose(ref, lib, rtol=1e-12)
    rep = O.reduce_fixed_order_fp32(L, 1, src)
    assert np.all(np.abs(rep - ref) <= 1e-6 * np.abs(ref))


def test_reduce_broadcast_dedup():
    """duplicated (zero-column) data is reduced once, not twice."""
    L = O.blocked([8, 16], [1, 2], [4, 8], [4, 1], [1, 0])      # 32 rows of slots for 8 rows: i-broadcast
    L = O.Layout(L.in_dims, L.out_dims, L.bases)
    assert any(c == 0 for c in L.cols)
    rng = np.random.default_rng(3)
    T = rng.random(128, dtype=np.float32)
    src = O.pack(L, T)
    rep = O.reduce_fixed_order_fp32(L, 1, src)
    ref = T.astype(np.float64).reshape(8, 16).sum(axis=1)
    assert np.allclose(rep, ref, rtol=1e-6)


def _reduce_rows(L, rows):
    """O11 replica applied to the logical [n_rows, K] tensor `rows` packed under L."""
    T = np.asarray(rows, dtype=np.float32).reshape(-1)
    return O.reduce_fixed_order_fp32(L, 1, O.pack(L, T))


@pytest.mark.parametrize("which", ["blocked_row", "blocked_col"])
def test_reduce_order_golden(which):
    """Pin (tests/golden/reduce_order.json, hand-derived under IEEE binary32 RN-even):
    the fixed order of reading R-reduce gives the expected fp32 bits on rows whose sum
    depends on the order, under two layouts that place the axis bits on different
    hardware levels (registers first vs lanes first)."""
    g = load("reduce_order.json")
    u = np.float32(2.0 ** -24)
    rows = [np.array(c["x_in_u"], dtype=np.float64) * float(u) for c in g["cases"]]
    L = {"blocked_row": O.blocked([4, 8], [1, 2], [4, 8], [1, 1], [1, 0]),
         "blocked_col": O.blocked([4, 8], [2, 1], [2, 16], [1, 1], [0, 1])}[which]
    out = _reduce_rows(L, rows)
    for c, got in zip(g["cases"], out):
        assert "%08x" % int(np.float32(got).view(np.uint32)) == c["expected_hex"], c["name"]
        for other in c["other_orders_hex"].values():
            assert other != c["expected_hex"]          # the case really separates orders


def _pairwise(x):
    """Textbook recursive pairwise summation in fp32 (Higham, Accuracy and Stability
    of Numerical Algorithms, §4.2): S(x) = S(x[:n/2]) + S(x[n/2:])."""
    if len(x) == 1:
        return np.float32(x[0])
    h = len(x) // 2
    return np.float32(_pairwise(x[:h]) + _pairwise(x[h:]))


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_reduce_order_is_recursive_pairwise(family):
    """Pin: the replica equals the recursive pairwise sum of each in-tile row segment
    (a top-down formulation of the same order), on [128, 128]-tile layouts of config 4
    with adversarial magnitudes (1 followed by tiny values, so that the order matters)."""
    rng = np.random.default_rng(11)
    L = L_of(W.c4("reduce", family, n_i=7, n_j=8))      # [128, 256], K = 128
    T = rng.random((128, 256), dtype=np.float32) * np.float32(2.0 ** -22)
    T[:, ::128] = 1.0
    got = O.reduce_fixed_order_fp32(L, 1, O.pack(L, T.reshape(-1))).reshape(128, 2)
    for r in range(0, 128, 7):
        for q in range(2):
            ref = _pairwise(list(T[r, q * 128:(q + 1) * 128]))
            assert got[r, q].view(np.uint32) == ref.view(np.uint32), (r, q)
    # the order matters on these rows: a sequential fp32 sum differs somewhere
    seq = np.array([np.float32(sum(np.float32(v) for v in T[r, :128])) for r in range(0, 128, 7)])
    assert np.any(seq.view(np.uint32) != got[::7, 0].view(np.uint32))


def test_reduce_order_layout_independent():
    """Invariant of reading R-reduce: the replica's bits depend on the logical tensor
    only — the MMA-accumulator and blocked layouts of config 4 give identical bits."""
    rng = np.random.default_rng(12)
    La = L_of(W.c4("reduce", "mma", n_i=8, n_j=8))
    Lb = L_of(W.c4("reduce", "blocked", n_i=8, n_j=8))
    T = (rng.random(1 << 16, dtype=np.float32) * np.float32(3.0)).astype(np.float32)
    ra = O.reduce_fixed_order_fp32(La, 1, O.pack(La, T))
    rb = O.reduce_fixed_order_fp32(Lb, 1, O.pack(Lb, T))
    assert np.array_equal(ra.view(np.uint32), rb.view(np.uint32))


def test_distributed_rank_slices_concatenate():
    """O12: the per-rank slices of B, for config-5 layouts at small size, are the
    column shards of the logical tensor (an all_to_all of row shards)."""
    rng = np.random.default_rng(1006)
    n = 4
    for p in (1, 2):
        A, B = (L_of(s) for s in W.c5(p, n=n))
        T = gen.random_bits(rng, 1 << (2 * n), 2)
        P = 1 << p
        M = T.reshape(1 << n, 1 << n)
        for r in range(P):
            got = O.convert_distributed_rank(A, B, T, r)
            cols = M[:, r * (16 // P):(r + 1) * (16 // P)]
            assert np.array_equal(got, cols.reshape(-1))


@pytest.mark.parametrize("bits", [16, 8, 32])
def test_oracle_mma_operand_matches_ptx(bits):
    """Prop 9.2 operand tiles in the oracle vs the PTX m16n8kK A / B
    fragment formulas [HW] (g = lane/4, t = lane%4, e = 32/bits elements per register):
    A: row = g + 8((i/e)%2), col = e·t + i%e + 4e·(i/(2e)); B: k = e·t + i%e + 4e·(i/e), n = g."""
    e = 32 // bits
    K = 8 * e
    A = O.mma_operand(False, (16, K), bits)
    B = O.mma_operand(True, (K, 8), bits)
    for h in range(1 << A.d_in):
        i, lane = h & ((1 << A.dim_bits("reg").__len__()) - 1), h >> len(A.dim_bits("reg"))
        g, t = lane // 4, lane % 4
        assert O.logical_coords(A.out_dims, O.apply(A, h)) == (g + 8 * ((i // e) % 2), e * t + i % e + 4 * e * (i // (2 * e)))
    for h in range(1 << B.d_in):
        i, lane = h & ((1 << len(B.dim_bits("reg"))) - 1), h >> len(B.dim_bits("reg"))
        g, t = lane // 4, lane % 4
        assert O.logical_coords(B.out_dims, O.apply(B, h)) == (e * t + i % e + 4 * e * (i // e), g)


# ----------------------------------------------------------------------------- GV6-GV8
def _flat(expr, j_bits):
    """'j3^i3' -> flat logical value (j_k = 2^k, i_k = 2^(k + j_bits))."""
    v = 0
    for term in expr.split("^"):
        k = int(term[1:])
        v ^= 1 << (k if term[0] == "j" else k + j_bits)
    return v


def test_gv6_config1_swizzle_columns():
    """GV6 (hand derivation of P:406-426 on Fig. 1 A -> B, tests/golden/derived_gv6_gv8.json):
    Vec = [j0, i0], Bank = [j1, j2, j3], Seg = H = [j1^i1, j2^i2, j3^i3], C empty."""
    g = load("derived_gv6_gv8.json")["GV6_config1"]
    sw = O.optimal_swizzle(L_of(W.C1_A), L_of(W.C1_B), 4)
    for key in ("Vec", "Bank", "Seg"):
        assert sw[key] == [_flat(e, g["j_bits"]) for e in g[key]], key
    assert sw["C"] == []


def test_gv7_config2_shuffle_sets():
    """GV7 (hand derivation of P:375-387 on config 2): V = [j0], I empty, E, F ascending,
    G = {e_i ^ f_i}, |R| = 6 -> 64 rounds."""
    g = load("derived_gv6_gv8.json")["GV7_config2"]
    sa, sb = W.c2(0)
    s = O.shuffle_sets(L_of(sa), L_of(sb), 2)
    for key in ("V", "I", "E", "F", "G"):
        assert s[key] == [_flat(e, g["j_bits"]) for e in g[key]], key
    assert len(s["R"]) == g["R_size"] and s["rounds"] == g["rounds"]


def test_gv8_config3_swizzle_and_offsets():
    """GV8 (hand derivation of P:406-426 on config 3): the swizzle columns, and the
    element offsets of eight logical points under the smem layout (offset bits Vec,
    Bank, Seg in that order) — S^{-1}(i, j)."""
    g = load("derived_gv6_gv8.json")["GV8_config3"]
    sa, sb = W.c3(0)
    A3, B3 = L_of(sa), L_of(sb)
    sw = O.optimal_swizzle(A3, B3, 2)
    for key in ("Vec", "Bank", "Seg"):
        assert sw[key] == [_flat(e, g["j_bits"]) for e in g[key]], key
    S = O.smem_layout_from_swizzle(sw, A3.out_dims)
    for (i, j), off in g["offsets"]:
        x = np.array([(i << g["j_bits"]) | j], dtype=np.uint64)
        assert int(O.apply_inverse_all(S, x)[0]) == off, (i, j)


# ----------------------------------------------------------------------------- O13 scan
@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_scan_fp64_is_cumsum_per_tile(family):
    """O13 fp64 reference against a hand loop: every output is the sum of its tile's
    axis prefix (brute force over a few points), computed without numpy.cumsum."""
    OL = L_of(W.c4("reduce", family, n_i=8, n_j=8))
    rng = np.random.default_rng(21)
    T = rng.random(1 << OL.d_out)
    src = O.pack(OL, T)
    out = O.scan_ref_fp64(OL, 1, src)
    x_of_h = O.image_table(OL).astype(np.int64)
    for h in rng.integers(0, src.size, size=64):
        x = int(x_of_h[h])
        i, j = x >> 8, x & 255
        j0 = j & ~127
        want = sum(T[(i << 8) | jj] for jj in range(j0, j + 1))
        assert abs(out[h] - want) <= 1e-12 * max(1.0, want)


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_scan_fp32_recurrence_exact_on_integers(family):
    """O13 fp32 bit-doubling recurrence: on integer-valued inputs every partial sum is
    exact in fp32 (< 2^24), so it must equal the integer cumulative sum exactly — any
    wrong partner index, step order or tile boundary fails."""
    OL = L_of(W.c4("reduce", family, n_i=8, n_j=8))
    rng = np.random.default_rng(22)
    T = rng.integers(0, 1000, size=1 << OL.d_out).astype(np.float32)
    src = O.pack(OL, T)
    got = O.scan_bitdoubling_fp32(OL, 1, src)
    want = O.scan_ref_fp64(OL, 1, src)
    assert np.array_equal(got.astype(np.float64), want)


def test_scan_fp32_recurrence_within_bound():
    """On U[0,1) inputs the recurrence (depth K_bits = 7 additions per element at most)
    stays within 7 * 2^-24 relative of the fp64 prefix sums."""
    OL = L_of(W.c4("reduce", "mma", n_i=8, n_j=8))
    src = O.pack(OL, np.random.default_rng(23).random(1 << OL.d_out, dtype=np.float32))
    got = O.scan_bitdoubling_fp32(OL, 1, src).astype(np.float64)
    ref = O.scan_ref_fp64(OL, 1, src)
    assert np.all(np.abs(got - ref) <= 7 * 2.0 ** -24 * np.abs(ref) + 1e-30)


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_reduce_max_min_closed_form(family):
    """max / min reductions (O11 with another op): on T[x] = x (the logical flat index,
    exact in fp64) the max over a [.., K] in-tile row is its last index and the min its
    first — a closed form independent of any layout arithmetic."""
    L = L_of(W.c4("reduce", family, n_i=8, n_j=8))     # [256, 256] in [128, 128] tiles
    n = 1 << L.d_in
    T = np.arange(n, dtype=np.float64)
    src = O.pack(L, T)
    rows = np.arange(256)[:, None] * 256 + np.arange(2)[None, :] * 128
    assert np.array_equal(O.reduce_ref_fp64(L, 1, src, "max"), (rows + 127).reshape(-1))
    assert np.array_equal(O.reduce_ref_fp64(L, 1, src, "min"), rows.reshape(-1))


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_scan_max_min_closed_form(family):
    """Running max / min scans: on T[x] = -x (decreasing along every row) the running
    max of a [.., K] in-tile row is its first element and the running min the element
    itself; on T[x] = x the other way round."""
    L = L_of(W.c4("reduce", family, n_i=8, n_j=8))     # [256, 256] in [128, 128] tiles
    n = 1 << L.d_in
    x = np.arange(n, dtype=np.float64)
    first = (x // 128) * 128                            # first index of x's in-tile row
    for T, mx, mn in ((-x, -first, -x), (x, x, first)):
        src = O.pack(L, T)
        assert np.array_equal(O.scan_ref_fp64(L, 1, src, "max"), O.pack(L, mx))
        assert np.array_equal(O.scan_ref_fp64(L, 1, src, "min"), O.pack(L, mn))


# ----------------------------------------------------------------------------- N2 TMEM

# CUTLASS SM100 TMEM_LOAD copy traits (flashinfer/data/cutlass/include/cute/atom/
# copy_traits_sm100.hpp, Copy_Traits<SM100_TMEM_LOAD_<dp>dp<bits>b<num>x>): the vendor's
# own description of each tcgen05.ld fragment as a CuTe layout
#   DstLayout: (thread, value bit) -> i,   ValID: i -> (bit = i % BITS, data path = i // BITS)
# written here as (thread shape, thread stride, value shape, value stride, BITS).
CUTE_TMEM_LOAD = {
    ("32x32b", 1): ((32,), (32,), (32,), (1,), 32),
    ("32x32b", 2): ((32,), (64,), (64,), (1,), 64),
    ("16x64b", 1): ((2, 2, 8), (512, 32, 64), (32,), (1,), 64),
    ("16x64b", 2): ((2, 2, 8), (1024, 32, 128), (32, 2), (1, 64), 128),
    ("16x128b", 1): ((4, 8), (32, 128), (32, 2), (1, 1024), 128),
    ("16x128b", 2): ((4, 8), (32, 256), (32, 2, 2), (1, 2048, 128), 256),
    ("16x256b", 1): ((4, 8), (64, 256), (64, 2), (1, 2048), 256),
    ("16x256b", 2): ((4, 8), (64, 512), (64, 2, 2), (1, 4096, 256), 512),
}


def _cute(shape, stride, lin):
    """CuTe layout function: colexicographic coordinates of `lin` dotted with stride."""
    out = 0
    for sz, st in zip(shape, stride):
        out += (lin % sz) * st
        lin //= sz
    return out


@pytest.mark.parametrize("key", sorted(CUTE_TMEM_LOAD))
def test_tmem_ld_matches_cutlass_traits(key):
    """N2: the oracle's tcgen05.ld fragment layouts (one warp, one load) equal the
    CUTLASS SM100 TMEM_LOAD traits at every (thread, register): register r holds value
    bits [32r, 32r + 32) of the thread, i.e. TMEM row dp and 32-bit column bit // 32."""
    shape, num = key
    tsh, tst, vsh, vst, BITS = CUTE_TMEM_LOAD[key]
    N = BITS // 32
    L = O.tmem_ld(shape, 128, N)
    nregs = int(np.prod(vsh)) // 32
    for t in range(32):
        for r in range(nregs):
            i = _cute(tsh, tst, t) + _cute(vsh, vst, 32 * r)
            dp, col = i // BITS, (i % BITS) // 32
            h = r | (t << L.dim_bits("lane")[0])
            assert O.apply(L, h) == (dp << (N.bit_length() - 1)) | col, (key, t, r)


@pytest.mark.parametrize("shape", ["32x32b", "16x64b", "16x128b", "16x256b"])
def test_n2_tmem_config_tables_are_the_fragments(shape):
    """The literal workload tables of N2 (workloads/configs.py) are the oracle's
    tcgen05.ld fragment layouts (pinned to CUTLASS above) on every tile."""
    sa, _ = W.n2_tmem(shape, nb=1)
    L = L_of(sa)
    F = O.tmem_ld(shape, 128, 128)
    assert [c & ((1 << 14) - 1) for c in L.cols[:F.d_in]] == F.cols


@pytest.mark.parametrize("bits", [8, 16])
def test_n2_acc_to_lhs_tables(bits):
    """The chained-GEMM tables are the oracle's Prop 9.2 accumulator (m64n64, 4 warps
    along M) and lhs operand (m64 x k64, `bits`-bit elements) layouts."""
    sa, sb = W.n2_acc_to_lhs(bits, nb=1)
    A, B = L_of(sa), L_of(sb)
    acc = O.mma_acc((64, 64), 4)
    lhs = O.mma_operand(False, (64, 64), bits, warps_m=4)
    m = (1 << 12) - 1
    assert [c & m for c in A.cols[:acc.d_in]] == acc.cols
    assert [c & m for c in B.cols[:lhs.d_in]] == lhs.cols
    assert O.classify(O.Layout(*W.spec_to_bases(W.n2_acc_to_lhs(bits, nb=0)[0])),
                      O.Layout(*W.spec_to_bases(W.n2_acc_to_lhs(bits, nb=0)[1]))) == \
        ("NOOP" if bits == 16 else "SHUFFLE")
