"""CPU tests of libll.so: the C ABI loads and exports every declared symbol; the
host F2 algebra and the planner agree with the oracle; the specialised plans'
schedules (emulated on the host with the same tables the kernels are compiled
from) reproduce the oracle's conversion; swizzles are bank-conflict free under the
oracle's Lemma 9.4 model; the kernel templates compile for sm_100a (NVRTC)."""
import ctypes
import os
import re

import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def both(spec):
    return ll.Layout.from_spec(spec), O.Layout(*W.spec_to_bases(spec))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "ll.h")).read()
    names = set(re.findall(r"^\s*(?:ll_status|void|const char\*)\s+(ll_\w+)\s*\(", hdr, re.M))
    assert len(names) >= 30
    lib = ctypes.CDLL(ll.library_path())
    missing = [n for n in sorted(names) if not hasattr(lib, n)]
    assert not missing, missing


def test_layout_roundtrip_and_apply():
    L, OL = both(W.C1_A)
    assert L.cols() == OL.cols
    for h in range(256):
        coords = O.hw_coords(OL.in_dims, h)
        assert L.apply(coords) == O.logical_coords(OL.out_dims, O.apply(OL, h))
    # predicates are properties of the matrix: a permutation matrix satisfies both
    # Def 4.10 and Def 4.14
    assert L.props() == dict(surjective=O.is_surjective(OL), injective=O.is_injective(OL),
                             distributed=O.is_distributed(OL), memory=O.is_memory(OL))


def test_algebra_vs_oracle_random():
    rng = np.random.default_rng(12)
    for _ in range(60):
        d_out = int(rng.integers(1, 6))
        d_in = int(rng.integers(d_out, 9))
        cols = gen.random_surjective_cols(rng, d_out, d_in)
        OL = O.layout_from_cols([("h", d_in)], [("x", d_out)], cols)
        L = ll.Layout([("h", d_in)], [("x", d_out)], {"h": [(c,) for c in cols]})
        # right inverse (Def 4.5): equals the oracle's brute-force min-index preimage
        Li = L.invert()
        first = O.preimage_min(OL)
        assert [b[0] for b in Li.bases()] == [int(first[1 << t]) for t in range(d_out)]
        # kernel dimension
        assert len(L.kernel_basis()) == d_in - d_out
        # compose with a random map (Def 4.2)
        d2 = int(rng.integers(1, 6))
        c2 = [int(x) for x in rng.integers(0, 1 << d2, size=d_out)]
        OM = O.layout_from_cols([("x", d_out)], [("y", d2)], c2)
        M = ll.Layout([("x", d_out)], [("y", d2)], {"x": [(c,) for c in c2]})
        assert M.compose(L).cols() == O.compose(OM, OL).cols
        p = L.props()
        assert p["surjective"] and p["injective"] == (d_in == d_out)


def test_product_and_left_division_vs_oracle():
    OA = O.blocked([4, 4], [2, 2], [2, 2], [1, 1], [1, 0])
    OB = O.blocked([8, 4], [1, 2], [4, 2], [2, 1], [1, 0])
    OA = O.Layout(OA.in_dims, [("d0", 2), ("d1", 2)], OA.bases)
    A = ll.Layout(OA.in_dims, OA.out_dims, OA.bases)
    B = ll.Layout(OB.in_dims, OB.out_dims, OB.bases)
    P = A.product(B)
    OP = O.product(OA, OB)
    assert P.cols() == OP.cols
    assert P.left_divide(A).cols() == OB.cols
    with pytest.raises(ll.LLError):
        P.left_divide(B)


def test_errors():
    A, _ = both(W.C1_A)
    B2, _ = both(W.c2(0)[0])
    with pytest.raises(ll.LLError, match="DIM_MISMATCH"):
        ll.ll_plan_convert(A, B2, 4)
    N = ll.Layout([("offset", 3)], [("x", 3)], {"offset": [(1,), (2,), (3,)]})
    with pytest.raises(ll.LLError, match="NOT_SURJECTIVE"):
        ll.ll_plan_convert(N, N, 4)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_plan_convert(A, A, 3)
    with pytest.raises(ll.LLError):
        ll.Layout([("reg", 1)], [("x", 1)], {"reg": [(2,)]})


@pytest.mark.parametrize("mvb", [3, 24, 32, 64, -4])
def test_max_vec_bytes_validated(mvb):
    """max_vec_bytes outside {0, 1, 2, 4, 8, 16} is rejected at plan time by every
    planner (no ld/st instruction is wider than 16 B): no plan silently
    falls back to byte loads."""
    A, _ = both(W.C1_A)
    B, _ = both(W.C1_B)
    L = ll.Layout.from_spec(W.c4("reduce", "mma", n_i=7, n_j=7))
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_plan_convert(A, B, 4, max_vec_bytes=mvb)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_plan_gather(ll.Layout.from_spec(W.c4("gather", "mma", n_i=7, n_j=5)), 1, 4, max_vec_bytes=mvb)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_plan_reduce(L, 1, max_vec_bytes=mvb)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_plan_scan(L, 1, max_vec_bytes=mvb)


@pytest.mark.parametrize("mvb", [1, 2, 4, 8, 16])
def test_max_vec_bytes_accepted(mvb):
    A, _ = both(W.C1_A)
    B, _ = both(W.C1_B)
    p = ll.ll_plan_convert(A, B, 4, max_vec_bytes=mvb)
    assert p.buffer_bytes() == (1024, 1024, 0)


def test_buffer_sizes_checked_before_launch():
    """The execution wrappers compare tensor sizes with ll_plan_buffer_bytes and raise
    before any pointer reaches the library (CPU tensors: nothing is launched)."""
    import torch
    A, _ = both(W.C1_A)
    B, _ = both(W.C1_B)
    p = ll.ll_plan_convert(A, B, 4)
    ok = torch.empty(256, dtype=torch.int32)
    small = torch.empty(255, dtype=torch.int32)
    with pytest.raises(ll.LLError, match="src"):
        ll.ll_convert(small, ok, p)
    with pytest.raises(ll.LLError, match="dst"):
        ll.ll_convert(ok, torch.empty(128, dtype=torch.int16), p)
    L = ll.Layout.from_spec(W.c4("gather", "mma", n_i=7, n_j=5))
    g = ll.ll_plan_gather(L, 1, 4)
    n = 1 << 12
    assert g.buffer_bytes() == (4 * n, 4 * n, 4 * n)
    with pytest.raises(ll.LLError, match="idx"):
        ll.ll_gather(torch.empty(n, dtype=torch.float32), torch.empty(n // 2, dtype=torch.int32),
                     torch.empty(n, dtype=torch.float32), g)
    R = ll.ll_plan_reduce(ll.Layout.from_spec(W.c4("reduce", "mma", n_i=7, n_j=7)), 1)
    assert R.buffer_bytes() == (4 << 14, 4 * R.out_elems(), 0)
    with pytest.raises(ll.LLError, match="dst"):
        ll.ll_reduce(torch.empty(1 << 14), torch.empty(R.out_elems() - 1), R)


@pytest.mark.parametrize("cfg", ["c1", "c2", "c3"])
def test_planner_class_matches_oracle_configs(cfg):
    sa, sb = {"c1": (W.C1_A, W.C1_B), "c2": W.c2(0), "c3": W.c3(0)}[cfg]
    A, OA = both(sa)
    B, OB = both(sb)
    assert ll.ll_plan_convert(A, B, 4).cls == O.classify(OA, OB)


def test_planner_class_matches_oracle_exhaustive_sample():
    """E1 (sampled): random relabelings B of Fig. 1's space, with and without
    broadcast columns; the planner's class equals the existential class O7."""
    rng = np.random.default_rng(31)
    A, OA = both(W.C1_A)
    hw = [("reg", 2), ("lane", 5), ("warp", 1)]
    for _ in range(300):
        sb = gen.random_distributed(rng, W.C1_OUT, hw)
        B, OB = both(sb)
        assert ll.ll_plan_convert(A, B, 4).cls == O.classify(OA, OB)
    out7 = [("i", 3), ("j", 4)]
    for _ in range(300):
        sa = gen.random_distributed(rng, out7, hw, zero_ok=["reg", "warp"])
        sb = gen.random_distributed(rng, out7, hw, zero_ok=["lane", "reg"])
        A7, OA7 = both(sa)
        B7, OB7 = both(sb)
        assert ll.ll_plan_convert(A7, B7, 4).cls == O.classify(OA7, OB7)


def _sim_check(sa, sb, w, seed, **opts):
    A, OA = both(sa)
    B, OB = both(sb)
    plan = ll.ll_plan_convert(A, B, w, **opts)
    rng = np.random.default_rng(seed)
    T = gen.random_bits(rng, 1 << OA.d_out, w)
    src = O.pack(OA, T)
    d = plan.describe()
    if d["exec"] != "tile":
        return d
    got = plan.simulate(src, 1 << OB.d_in)
    assert np.array_equal(got, O.convert(OA, OB, src)), d
    return d


@pytest.mark.parametrize("force", [None, "SMEM"])
@pytest.mark.parametrize("sigma", ["coalesced", "faithful"])
def test_simulated_schedule_configs(force, sigma):
    for sa, sb, w in [(W.C1_A, W.C1_B, 4), (*W.c1_batched(5), 4), (*W.c2(1), 2), (*W.c3(1), 2), (*W.c3b(1), 2)]:
        d = _sim_check(sa, sb, w, 1, force_class=force, sigma=sigma)
        assert d["exec"] == "tile"
        if force == "SMEM":
            assert d["tile"]["xchg"] == "smem"


def test_simulated_schedule_random_distributed():
    rng = np.random.default_rng(77)
    out = [("i", 5), ("j", 5)]
    hw = [("reg", 2), ("lane", 5), ("warp", 3)]
    seen = set()
    for case in range(80):
        sa = gen.random_distributed(rng, out, hw)
        sb = gen.random_distributed(rng, out, hw)
        w = [1, 2, 4, 8][case % 4]
        d = _sim_check(sa, sb, w, case)
        seen.add((d["class"], d.get("tile", {}).get("xchg")))
    assert ("SMEM", "smem") in seen


def test_simulated_schedule_regperm_shuffle_classes():
    """REGPERM and SHUFFLE class pairs built by permuting only
    register bits / register+lane bits of a random layout."""
    rng = np.random.default_rng(8)
    out = [("i", 5), ("j", 5)]
    hw = [("reg", 3), ("lane", 5), ("warp", 2)]
    for case in range(40):
        sa = gen.random_distributed(rng, out, hw)
        ins = dict(sa["in"])
        if case % 2 == 0:
            regs = list(ins["reg"])
            rng.shuffle(regs)
            sb = {"out": out, "in": [("reg", regs), ("lane", ins["lane"]), ("warp", ins["warp"])]}
            want = "REGPERM"
        else:
            pool = list(ins["reg"]) + list(ins["lane"])
            rng.shuffle(pool)
            sb = {"out": out, "in": [("reg", pool[:3]), ("lane", pool[3:]), ("warp", ins["warp"])]}
            want = "SHUFFLE"
        A, OA = both(sa)
        B, OB = both(sb)
        if O.classify(OA, OB) != want:
            continue
        for w in (2, 4):
            d = _sim_check(sa, sb, w, case, sigma="faithful")
            assert d["class"] == want


def test_simulated_schedule_cta_class():
    rng = np.random.default_rng(5)
    out = [("i", 6), ("j", 6)]
    name = lambda k: f"j{k}" if k < 6 else f"i{k - 6}"
    for case in range(20):
        sa = {"out": out, "in": [("offset", [name(k) for k in rng.permutation(12)])]}
        sb = {"out": out, "in": [("offset", [name(k) for k in rng.permutation(12)])]}
        d = _sim_check(sa, sb, [1, 2, 4][case % 3], case)
        assert d["class"] in ("CTA", "NOOP")


def test_swizzle_plans_conflict_free_under_oracle_model():
    """The planner's smem layout (Vec, Bank, Seg) gives the ideal number of wavefronts
    for the store (L_ld) and load (L_st) sides under the oracle's simulator."""
    for sa, sb, w in [(W.C1_A, W.C1_B, 4), (*W.c2(0), 2), (*W.c3(0), 2), (*W.c3b(0), 2)]:
        A, OA = both(sa)
        B, OB = both(sb)
        t = ll.ll_plan_convert(A, B, w, force_class="SMEM").describe()["tile"]
        out = OA.out_dims
        mk = lambda cols: O.layout_from_cols([("reg", t["R"]), ("lane", 5), ("warp", t["warp_bits"])], out, cols)
        Lld, Lst = mk(t["L_ld"]), mk(t["L_st"])
        S = O.layout_from_cols([("offset", t["n"])], out, t["Vec"] + t["Bank"] + t["Seg"])
        assert O.is_memory(S) or O.is_surjective(S)
        for L, instr, word in ((Lld, t["smem_store"], t["mat_word_ld"]), (Lst, t["smem_load"], t["mat_word_st"])):
            if "matrix" in instr:
                wf, ideal = O.smem_matrix_wavefronts(S, L, w, [L.cols[b] for b in word], trans=".trans" in instr)
            else:
                wf, ideal = O.smem_wavefronts(S, L, w, t["Vec"])
            assert wf == ideal
        assert t["wavefronts_st"] + t["wavefronts_ld"] == t["ideal_wavefronts"]


def test_shuffle_plan_invariants_config2():
    """O9: rounds = 2^{(n_reg+5) - |V| - |I| - |G|}; G = {e_i ^ f_i} with E, F
    ascending; one 32-bit unit per lane per round."""
    A, _ = both(W.c2(0)[0])
    B, _ = both(W.c2(0)[1])
    t = ll.ll_plan_convert(A, B, 2).describe()["tile"]
    assert t["xchg"] == "shuffle"
    assert t["rounds"] == 1 << ((t["R"] + 5) - len(t["V"]) - len(t["I"]) - len(t["G"]))
    assert t["E"] == sorted(t["E"]) and t["F"] == sorted(t["F"])
    assert t["G"] == [e ^ f for e, f in zip(t["E"], t["F"])]
    assert t["unit_elems"] * 2 == 4


def test_kernels_compile_for_sm100a():
    """NVRTC specialisation of each kernel family for sm_100a (no GPU needed)."""
    for sa, sb, w, fc in [(*W.c2(16), 2, None), (*W.c3(14), 2, None), (W.C1_A, W.C1_B, 4, "SMEM")]:
        A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
        p = ll.ll_plan_convert(A, B, w, force_class=fc)
        p.precompile()
        assert "ll_tile_kernel" in p.source()
    L = ll.Layout.from_spec(W.c4("gather", "mma"))
    ll.ll_plan_gather(L, 1, 4).precompile()
    L = ll.Layout.from_spec(W.c4("reduce", "blocked"))
    ll.ll_plan_reduce(L, 1).precompile()


def test_device_entry_fails_loudly_without_gpu():
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    A, B = ll.Layout.from_spec(W.C1_A), ll.Layout.from_spec(W.C1_B)
    p = ll.ll_plan_convert(A, B, 4)
    with pytest.raises(ll.LLError, match="CUDA"):
        ll.ll_convert(1 << 20, 2 << 20, p, stream=0)
    with pytest.raises(ll.LLError, match="CUDA"):
        ll.ll_plan_autotune(A, B, 4, 1 << 20, 2 << 20, stream=0)


# ---------------------------------------------------------------- layout families
@pytest.mark.parametrize("args", [
    ([16, 16], [2, 2], [4, 8], [2, 1], [1, 0]),
    ([128, 128], [8, 8], [2, 16], [4, 1], [1, 0]),
    ([256, 128], [1, 8], [2, 16], [4, 1], [1, 0]),
    ([256, 128], [8, 1], [32, 1], [1, 4], [0, 1]),
    ([8, 8], [1, 1], [4, 8], [2, 1], [1, 0]),          # broadcast
    ([4, 8, 16], [1, 2, 2], [2, 4, 4], [1, 2, 2], [2, 1, 0]),
])
def test_blocked_family_matches_oracle(args):
    L = ll.ll_layout_blocked(*args)
    OL = O.blocked(*args)
    assert L.cols() == OL.cols and L.in_dims == OL.in_dims


def test_blocked_is_fig1_A():
    """GV3 through the product's constructor: blocked([2,2],[4,8],[2,1],[1,0]) on
    16x16 has the columns of the P:140 matrix."""
    L = ll.ll_layout_blocked([16, 16], [2, 2], [4, 8], [2, 1], [1, 0])
    assert L.cols() == O.Layout(*W.spec_to_bases(W.C1_A)).cols


@pytest.mark.parametrize("M,N,wm", [(128, 128, 4), (64, 32, 4), (16, 8, 1), (128, 32, 4)])
def test_mma_acc_family_matches_oracle(M, N, wm):
    assert ll.ll_layout_mma_acc(M, N, wm).cols() == O.mma_acc([M, N], wm).cols


def test_mma_swizzle_family_matches_def411():
    for vec, pp, mp in [(8, 1, 8), (4, 2, 4), (8, 2, 4), (2, 1, 8)]:
        L = ll.ll_layout_mma_swizzle(6, 6, vec, pp, mp)
        assert L.props()["memory"]
        # the map is an involution: offset(i, j) = (i << 6) + Def 4.11 formula
        cols = L.cols()
        for i in range(64):
            for j in range(64):
                x = (i << 6) | j
                off = 0
                for k in range(12):
                    if (x >> k) & 1:
                        off ^= cols[k]
                assert off == (i << 6) + O.mma_swizzle_offset(i, j, vec, pp, mp)


def test_slice_family_matches_oracle():
    L = ll.ll_layout_blocked([16, 16], [2, 2], [4, 8], [2, 1], [1, 0])
    S = ll.ll_layout_slice(L, 1)
    OS = O.sliced(O.blocked([16, 16], [2, 2], [4, 8], [2, 1], [1, 0]), 1)
    assert S.cols() == OS.cols
    assert S.props()["surjective"] and not S.props()["injective"]


def test_contiguity_table3():
    """P:300-304 contiguity reproduces Table 3's Triton-Linear bitwidths
    on the blocked layouts of the fixture (layouts are a reading, G23)."""
    import json
    rows = json.load(open(os.path.join(ROOT, "tests", "golden", "table3_contiguity.json")))["rows"]
    for r in rows:
        L = ll.ll_layout_blocked(r["shape"], r["size_per_thread"], [4, 8], [4, 1], [1, 0])
        assert L.contiguity(r["dtype_bytes"]) * r["dtype_bytes"] * 8 == r["bits"], r
    # legacy Triton's fastest-dim-only rule would give 16 bits for [512,2] x f8
    L = ll.ll_layout_blocked([512, 2], [8, 2], [4, 8], [4, 1], [1, 0])
    assert L.cols()[0] == 1 and L.cols()[1] == 2   # j0 then i0: contiguous across dims


# ---------------------------------------------------------------- N2: operand / TMEM families
def _enum(L):
    """(reg, lane, warp) -> logical coords for every hardware index of L."""
    d = {}
    ins = L.in_dims
    nr, nl, nw = [dict(ins).get(k, 0) for k in ("reg", "lane", "warp")]
    for w in range(1 << nw):
        for l in range(1 << nl):
            for r in range(1 << nr):
                d[(r, l, w)] = L.apply([r, l, w][:len(ins)])
    return d


@pytest.mark.parametrize("bits", [16, 8, 32])
def test_mma_lhs_matches_ptx_fragment(bits):
    """Prop 9.2 lhs tile vs the PTX m16n8k{8,16,32} A fragment [HW]: element i of
    lane (g = lane/4, t = lane%4) at row g + 8·((i/e)%2), col e·t + i%e + 4e·(i/(2e)),
    e = 32/bits elements per 32-bit register."""
    e = 32 // bits
    K = 8 * e
    L = ll.ll_layout_mma_operand(0, 16, K, bits)
    for (r, lane, w), (row, col) in _enum(L).items():
        g, t = lane // 4, lane % 4
        assert row == g + 8 * ((r // e) % 2), (r, lane)
        assert col == e * t + r % e + 4 * e * (r // (2 * e)), (r, lane)


@pytest.mark.parametrize("bits", [16, 8, 32])
def test_mma_rhs_matches_ptx_fragment(bits):
    """Prop 9.2 rhs tile vs the PTX B fragment [HW]: element i at
    k = e·t + i%e + 4e·(i/e), n = g."""
    e = 32 // bits
    K = 8 * e
    L = ll.ll_layout_mma_operand(1, K, 8, bits)
    for (r, lane, w), (k, n) in _enum(L).items():
        g, t = lane // 4, lane % 4
        assert k == e * t + r % e + 4 * e * (r // e) and n == g, (r, lane)


def test_mma_acc_to_lhs_is_free():
    """The m16n8 fp32 accumulator of a 16x16 tile has the columns of the m16n8k16 bf16
    lhs operand (reg j0, i3, j3; lanes j1 j2 i0 i1 i2), so converting the accumulator
    (after a per-element downcast) into the next mma's A operand is NOOP — the register
    reuse FlashAttention exploits."""
    acc = ll.ll_layout_mma_acc(16, 16, 1)
    lhs = ll.ll_layout_mma_operand(0, 16, 16, 16)
    assert acc.cols() == lhs.cols()
    assert ll.ll_plan_convert(acc, lhs, 2).cls == "NOOP"


def test_wgmma_lhs_and_broadcast_warps():
    """wgmma lhs = mma lhs x id^{Wrp,0}_2; with warps along N the lhs is
    broadcast over those warps (zero columns)."""
    L = ll.ll_layout_mma_operand(0, 64, 16, 16, warps_m=4)
    c = L.cols()
    assert c[-2:] == [16 << 4, 16 << 5]          # warps -> i4, i5
    L2 = ll.ll_layout_mma_operand(0, 16, 16, 16, warps_m=1, warps_n=2)
    assert L2.cols()[-1] == 0 and L2.props()["surjective"] and not L2.props()["injective"]


def test_tmem_fragment_family():
    L = ll.ll_layout_tmem_32x32b(128, 64)
    for (r, lane, w), (row, col) in _enum(L).items():
        assert row == 32 * w + lane and col == r
    B = ll.ll_layout_blocked([128, 64], [1, 4], [2, 16], [4, 1], [1, 0])
    p = ll.ll_plan_convert(L, B, 4)
    assert p.cls == "SMEM"


def test_simulated_schedule_broadcast_layouts():
    """Rule (2) / broadcast: layouts with zero columns run in the
    specialised tile kernels — zero src bits are never read, zero dst bits become store
    replicas; the emulated schedule equals the oracle's conversion."""
    rng = np.random.default_rng(5)
    tiles = 0
    opts_z = [["reg", "lane"], ["lane", "warp"], ["reg", "warp", "block"], ["reg", "lane", "warp", "block"]]
    for case in range(120):
        out = [("i", 3 + case % 3), ("j", 4)]
        hw = [("reg", 3), ("lane", 5), ("warp", 2), ("block", 1)]
        sa = gen.random_distributed(rng, out, hw, zero_ok=opts_z[case % 4])
        sb = gen.random_distributed(rng, out, hw, zero_ok=opts_z[(case // 4) % 4])
        d = _sim_check(sa, sb, [1, 2, 4, 8][case % 4], case)
        tiles += d["exec"] == "tile"
    assert tiles >= 20


def test_exhaustive_fig1_all_40320():
    """E1, exhaustive: every bijective relabeling B of Fig. 1's 2^8 space
    (8! = 40320) against Fig. 1 A.  The planner's class equals the existential
    class oracle (O7, evaluated here through its level test on the pull map, vectorised
    over all B), and every specialised plan's emulated schedule reproduces the oracle's
    conversion pack_A(T) -> pack_B(T)."""
    import itertools
    A, OA = both(W.C1_A)
    T = gen.random_bits(np.random.default_rng(1001), 256, 4)
    src = O.pack(OA, T)
    hs = np.arange(256, dtype=np.int64)
    counts = {}
    unit = [1 << t for t in range(8)]
    hw_names = ["reg", "reg", "lane", "lane", "lane", "lane", "lane", "warp"]
    for case, perm in enumerate(itertools.permutations(range(8))):
        cols = [unit[p] for p in perm]
        OB = O.layout_from_cols(OA.in_dims, OA.out_dims, cols)
        B = ll.Layout(OB.in_dims, OB.out_dims, OB.bases)
        plan = ll.ll_plan_convert(A, B, 4)
        cls = plan.cls
        counts[cls] = counts.get(cls, 0) + 1
        if case % 97 == 0:       # the brute-force O7 on a 1/97 sample (it is slow)
            assert cls == O.classify(OA, OB), perm
        want = O.pack(OB, T)
        d = plan.describe()
        if d["exec"] == "tile":
            assert np.array_equal(plan.simulate(src, 256), want), perm
    assert sum(counts.values()) == 40320
    # bijective relabelings never broadcast: NOOP exactly once (B = A)
    assert counts.get("NOOP") == 1


@pytest.mark.parametrize("vec,pp,mp", [(8, 1, 8), (4, 2, 4), (8, 2, 4), (2, 1, 8), (1, 1, 8), (1, 2, 4)])
def test_swizzled_memory_layout_xor_copy(vec, pp, mp):
    """Row-major -> Def 4.11 mma-swizzled memory layout and back: the pull
    map has 2-bit columns; the planner runs it as a vectorised XOR-column copy kernel
    whose emulated schedule equals the oracle (and the Def 4.11 formula)."""
    m = n = 6
    rng = np.random.default_rng(vec * 100 + pp * 10 + mp)
    row = O.identity_memory([("i", m), ("j", n)])
    S = ll.ll_layout_mma_swizzle(m, n, vec, pp, mp)
    R = ll.Layout(row.in_dims, [("d0", m), ("d1", n)], {"offset": [((c >> n), c & ((1 << n) - 1)) for c in row.cols]})
    T = gen.random_bits(rng, 1 << (m + n), 2)
    for A, B in ((R, S), (S, R)):
        p = ll.ll_plan_convert(A, B, 2)
        assert p.describe()["exec"] == "tile"
        assert p.describe()["tile"]["vld"] == 3      # whole 16-byte vectors (in-vector XOR below)
        OA = O.layout_from_cols([("offset", m + n)], [("d0", m), ("d1", n)], A.cols())
        OB = O.layout_from_cols([("offset", m + n)], [("d0", m), ("d1", n)], B.cols())
        src = O.pack(OA, T)
        assert np.array_equal(p.simulate(src, 1 << (m + n)), O.convert(OA, OB, src))
    # the swizzled buffer holds element (i, j) at offset i*2^n + Def 4.11 offset
    p = ll.ll_plan_convert(R, S, 2)
    got = p.simulate(T, 1 << (m + n))
    for i in range(0, 64, 5):
        for j in range(0, 64, 3):
            assert got[(i << n) + O.mma_swizzle_offset(i, j, vec, pp, mp)] == T[(i << n) + j]


@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_random_memory_layouts_xor_copy_simulated(w):
    """R2 random memory layouts (Def 4.14: 1- or 2-bit columns) <-> row-major, d = 5..10:
    every XOR-copy tile plan's emulated schedule — with the kernel's own address
    arithmetic (thread part XOR tile base, register part XOR, vector element +i) —
    equals the oracle.  (A vector whose start another column reaches below bit v would
    be misaligned: the planner narrows v.)"""
    tiles = 0
    for d in range(5, 11):
        for seed in range(12):
            rng = np.random.default_rng(seed * 7 + d + 1000 * w)
            out = [("x", d)]
            OA = O.Layout([("offset", d)], out, {"offset": [[1 << k] for k in range(d)]})
            OB = O.layout_from_cols([("offset", d)], out, gen.random_memory_cols(rng, d))
            A = ll.Layout(OA.in_dims, OA.out_dims, OA.bases)
            B = ll.Layout(OB.in_dims, OB.out_dims, OB.bases)
            T = gen.random_bits(rng, 1 << d, w)
            for A_, B_, OA_, OB_ in ((A, B, OA, OB), (B, A, OB, OA)):
                p = ll.ll_plan_convert(A_, B_, w)
                if p.describe()["exec"] != "tile":
                    continue
                tiles += 1
                s = O.pack(OA_, T)
                assert np.array_equal(p.simulate(s, 1 << d), O.convert(OA_, OB_, s)), (d, seed)
    assert tiles >= 40


def test_planner_faithful_reproduces_gv6_gv8():
    """Under faithful σ (the kernel holds the data exactly as the paper's layouts do) the
    planner's swizzle and shuffle sets equal the hand derivations GV6-GV8 of the paper's
    constructions (tests/golden/derived_gv6_gv8.json).  The
    swizzle derivations use the vectorised ld/st.shared tile, so stmatrix /
    ldmatrix selection is switched off here (smem_instr="vec")."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "derived_gv6_gv8.json")))

    def flat(e, jb):
        v = 0
        for t in e.split("^"):
            v ^= 1 << (int(t[1:]) if t[0] == "j" else int(t[1:]) + jb)
        return v
    for key, (sa, sb), w, fields in [("GV6_config1", (W.C1_A, W.C1_B), 4, ("Vec", "Bank", "Seg")),
                                     ("GV8_config3", W.c3(0), 2, ("Vec", "Bank", "Seg")),
                                     ("GV7_config2", W.c2(0), 2, ("V", "I", "E", "F", "G"))]:
        p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w, sigma="faithful",
                               smem_instr="vec")
        t = p.describe()["tile"]
        for f in fields:
            assert t[f] == [flat(e, g[key]["j_bits"]) for e in g[key][f]], (key, f)
    assert t["rounds"] == g["GV7_config2"]["rounds"]


def test_scan_plans():
    """Scan plans (§8(f) N3): one step per in-tile axis bit; config 4's axis bits sit on
    registers and lanes (no shared memory), an axis over the warps adds the
    shared-memory exchange (one fp32 per thread and register)."""
    for fam in ("mma", "blocked"):
        d = ll.ll_plan_scan(ll.Layout.from_spec(W.c4("reduce", fam)), 1).describe()
        assert d["kind"] == "scan" and d["steps"] == 7 and len(d["axis_hw"]) == 7
        assert all(b < d["R"] + 5 for b in d["axis_hw"]) and d["smem_exchange_bytes"] == 0
        assert d["ctas"] == 1024
    spec = {"out": [("i", 5), ("j", 7)],
            "in": [("reg", ["j0", "j1", "j2"]), ("lane", ["i0", "i1", "i2", "i3", "i4"]), ("warp", ["j3", "j4", "j5", "j6"])]}
    d = ll.ll_plan_scan(ll.Layout.from_spec(spec), 1).describe()
    assert d["smem_exchange_bytes"] == 4 * 8 * 512


# ----------------------------------------------------------------------------- Thm 5.1
from tests._matrix_cases import MATRIX_CASES  # noqa: E402


def _check_matrix_plan(t, OA, w):
    """Oracle-side checks of an SMEM tile plan whose sides may use stmatrix / ldmatrix:
    the oracle's bank model (P:344 fragment semantics; raises unless every matrix row is
    16 contiguous bytes) counts the wavefronts the planner predicts for each side, and a
    non-transposed matrix side satisfies Thm 5.1 by the paper's left division (Def 4.4)
    after renaming the word registers first (P_Reg)."""
    out = OA.out_dims
    hw = [("reg", t["R"]), ("lane", 5), ("warp", t["warp_bits"])]
    S = O.layout_from_cols([("offset", t["n"])], out, t["Vec"] + t["Bank"] + t["Seg"])
    S_inv = O.right_inverse(S)
    k = (4 // w).bit_length() - 1
    for cols, instr, word, pred in ((t["L_ld"], t["smem_store"], t["mat_word_ld"], t["wavefronts_st"]),
                                    (t["L_st"], t["smem_load"], t["mat_word_st"], t["wavefronts_ld"])):
        L = O.layout_from_cols(hw, out, cols)
        if "matrix" not in instr:
            wf, ideal = O.smem_wavefronts(S, L, w, t["Vec"])
            assert wf == pred, instr
            continue
        wf, ideal = O.smem_matrix_wavefronts(S, L, w, [cols[b] for b in word], trans=".trans" in instr)
        assert wf == pred, instr
        if ".trans" in instr:
            continue
        # P_Reg: word registers first, then the rest in order
        regs = list(word) + [b for b in range(t["R"]) if b not in word]
        cols2 = [cols[b] for b in regs] + cols[t["R"]:]
        Moff = O.compose(S_inv, O.layout_from_cols(hw, out, cols2))       # hw -> offset
        T = O.Layout([("reg", k), ("lane", 2)], [("offset", k + 2)],
                     {"reg": [(1 << i,) for i in range(k)], "lane": [(1 << (k + i),) for i in range(2)]})
        O.left_divide(Moff, T)     # raises if the tile does not divide


@pytest.mark.parametrize("case", MATRIX_CASES, ids=[c[0] for c in MATRIX_CASES])
def test_matrix_tiles_literal_cases(case):
    """stmatrix / ldmatrix (.x1/.x2/.x4, .trans) selection on literal layout pairs:
    the expected instructions, the plan's schedule reproduces the oracle conversion,
    and the oracle's bank model / Thm 5.1 checks hold."""
    name, sa, sb, w, (want_st, want_ld) = case
    d = _sim_check(sa, sb, w, 3, sigma="faithful", force_class="SMEM")
    t = d["tile"]
    assert (t["smem_store"], t["smem_load"]) == (want_st, want_ld)
    assert t["wavefronts_st"] + t["wavefronts_ld"] == t["ideal_wavefronts"]
    _check_matrix_plan(t, both(sa)[1], w)


def test_matrix_tiles_on_paper_configs():
    """Thm 5.1 selection on the paper's layouts (faithful σ): the wgmma accumulator of
    config 2 (each thread 4 contiguous bytes, lanes 0,1 along j) is stored with
    stmatrix.x4 and the blocked side loaded with ld.shared.v4 — 16 instructions per
    thread per side instead of 32 with the common 8-byte register vector; config 3's
    blocked [1,8] side also goes through stmatrix (32 instead of 128: -75%, the Table 4
    kind of smem-instruction reduction).  Coalesced σ on config 3b widens the
    swizzle vector from 8 to 16 bytes with stmatrix."""
    cases = [(W.c2(0), 2, "faithful", 16, 32), (W.c3(0), 2, "faithful", 32, 128), (W.c3b(0), 2, "coalesced", None, None)]
    for (sa, sb), w, sigma, n_mat, n_vec in cases:
        # the automatic choice takes stmatrix for config 3 (4-byte common vector) and 3b;
        # config 2 (8-byte common vector under faithful σ) keeps the vectorised path
        # by the measured default and gets the matrix tiles on request
        auto = _sim_check(sa, sb, w, 4, sigma=sigma, force_class="SMEM")["tile"]
        assert ("stmatrix" in auto["smem_store"]) == (n_mat != 16)
        d = _sim_check(sa, sb, w, 4, sigma=sigma, force_class="SMEM", smem_instr="matrix")
        t = d["tile"]
        assert t["smem_store"] == "stmatrix.m8n8.x4.b16" and t["smem_load"] == "ld.shared.v4.b32", t
        assert (1 << len(t["Vec"])) * w == 16
        _check_matrix_plan(t, both(sa)[1], w)
        if n_mat:
            A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
            tv = ll.ll_plan_convert(A, B, w, sigma=sigma, force_class="SMEM", smem_instr="vec").describe()["tile"]
            assert t["smem_store_instrs"] == n_mat and tv["smem_store_instrs"] == n_vec


def test_matrix_tiles_random_layouts_simulated():
    """Random distributed pairs (R1) planned with smem_instr = "matrix": every matrix
    side is bit-exact in the host schedule emulation and passes the oracle checks."""
    rng = np.random.default_rng(344)
    out = [("i", 5), ("j", 5)]
    seen = set()
    for R in (1, 2, 3):
        hw = [("reg", R), ("lane", 5), ("warp", 5 - R)]
        for case in range(24):
            sa = gen.random_distributed(rng, out, hw)
            sb = gen.random_distributed(rng, out, hw)
            w = [1, 2, 4][case % 3]
            sigma = ("faithful", "coalesced")[case % 2]
            d = _sim_check(sa, sb, w, case, sigma=sigma, force_class="SMEM", smem_instr="matrix")
            t = d["tile"]
            _check_matrix_plan(t, both(sa)[1], w)
            seen.add(t["smem_store"].split(".")[0] + "/" + t["smem_load"].split(".")[0])
    assert {"stmatrix/ld", "st/ldmatrix"} <= seen, seen


def test_matrix_kernels_emit_stsm_ldsm_sass(tmp_path, monkeypatch):
    """The specialised sm_100a kernels really use the matrix instructions: SASS of the
    NVRTC cubins (cuobjdump, no GPU needed) holds STSM / LDSM (.MT88 = transposed)."""
    import shutil
    import subprocess
    cuobjdump = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cuobjdump):
        pytest.skip("cuobjdump not available")
    want = {"x1_mat_to_trans_b16": ("STSM.16.M88 ", "LDSM.16.MT88 "),
            "x2_mat_mat_b32": ("STSM.16.M88.2", "LDSM.16.M88.2"),
            "x4_mat_to_vec_b8": ("STSM.16.M88.4", "LDS.128"),
            "x4_trans_to_vec_b16": ("STSM.16.MT88.4", "LDS.128")}
    for name, sa, sb, w, _ in MATRIX_CASES:
        d = tmp_path / name
        d.mkdir()
        monkeypatch.setenv("LL_JIT_CACHE", str(d))
        ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w, sigma="faithful",
                           force_class="SMEM").precompile()
        (cubin,) = list(d.glob("*.cubin"))
        sass = subprocess.run([cuobjdump, "-sass", str(cubin)], capture_output=True, text=True, check=True).stdout
        sass = sass.replace(" ;", " ")
        for mnem in want[name]:
            assert mnem in sass, (name, mnem)


def test_env_hooks_force_class_and_log():
    """LL_FORCE_CLASS / LL_LOG (include/ll.h ENVIRONMENT) in a fresh process."""
    import subprocess
    import sys
    code = ("import sys; sys.path.insert(0, %r)\n"
            "import paper_conf_asplos_0001cgrnls0trm26_b200 as ll\n"
            "from workloads import configs as W\n"
            "sa, sb = W.c2(0)\n"
            "p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2)\n"
            "print(p.describe()['tile']['xchg'])\n") % os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, LL_FORCE_CLASS="smem", LL_LOG="1")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, check=True)
    assert r.stdout.strip() == "smem"
    assert r.stderr.startswith("[ll] plan {") and '"xchg":"smem"' in r.stderr
    env = {k: v for k, v in os.environ.items() if k not in ("LL_FORCE_CLASS", "LL_LOG")}
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, check=True)
    assert r.stdout.strip() == "shuffle" and "[ll] plan" not in r.stderr


@pytest.mark.parametrize("w", [1, 4, 8])
def test_swizzled_memory_layout_in_vector_xor_other_widths(w):
    """In-vector XOR copies for 1-, 4- and 8-byte elements (the bf16 case is above):
    16-byte vectors for every Def 4.11 parameter set, emulated schedule == oracle."""
    m = n = 6
    row = O.identity_memory([("i", m), ("j", n)])
    R = ll.Layout(row.in_dims, [("d0", m), ("d1", n)], {"offset": [((c >> n), c & ((1 << n) - 1)) for c in row.cols]})
    rng = np.random.default_rng(w)
    for vec, pp, mp in [(1, 1, 8), (2, 1, 8), (4, 2, 4), (8, 1, 8), (1, 2, 4)]:
        S = ll.ll_layout_mma_swizzle(m, n, vec, pp, mp)
        for A, B in ((R, S), (S, R)):
            p = ll.ll_plan_convert(A, B, w)
            t = p.describe()["tile"]
            assert (1 << t["vld"]) * min(w, 4) == 16
            OA = O.layout_from_cols([("offset", m + n)], [("d0", m), ("d1", n)], A.cols())
            OB = O.layout_from_cols([("offset", m + n)], [("d0", m), ("d1", n)], B.cols())
            src = O.pack(OA, gen.random_bits(rng, 1 << (m + n), w))
            assert np.array_equal(p.simulate(src, 1 << (m + n)), O.convert(OA, OB, src)), (vec, pp, mp)


def test_convert_host_refuses_xor_grids():
    """ll_convert_host chunks the batch by CTA tiles; a Def 4.11 swizzle's XOR grid
    (row bits XOR into column bits) indexes src by the global tile number, so the call
    is refused up front (LL_ERR_UNSUPPORTED) rather than computed per chunk."""
    import ctypes as C
    m = n = 10
    row = O.identity_memory([("i", m), ("j", n)])
    R = ll.Layout(row.in_dims, [("d0", m), ("d1", n)], {"offset": [((c >> n), c & ((1 << n) - 1)) for c in row.cols]})
    S = ll.ll_layout_mma_swizzle(m, n, 8, 16, 8)       # row bits 4-6 XOR into the columns
    p = ll.ll_plan_convert(R, S, 2)
    t = p.describe()["tile"]
    assert t["grid_dst_bit"] and t["n"] < n + 4     # row bit 4 is a grid bit
    h = np.zeros(1 << (m + n), dtype=np.uint16)
    dev = np.zeros(1 << 16, dtype=np.uint8)
    streams = (C.c_void_p * 1)(None)
    st = ll._lib.ll_convert_host(h.ctypes.data, h.ctypes.data, (dev.ctypes.data + 15) // 16 * 16, 1 << 15,
                                 p.handle, 1, streams)
    assert ll.STATUS[st] == "UNSUPPORTED"
    assert b"grid" in ll._lib.ll_last_error()


def test_comm_check_loopback_ok_and_null_invalid():
    """ll_comm_check (failure detection): loopback communicators have no NCCL state
    (LL_OK); a null handle is an invalid argument."""
    c = ll.Comm.loopback(4)
    c.check()
    assert ll.STATUS[ll._lib.ll_comm_check(None)] == "INVALID_ARG"


def test_linear_tiles_with_identical_dev_bits():
    """General memory layouts (R2) with the same `dev` bits in A and B: the class stays
    local (CTA), each rank's slice is planned as a linear tile over its local bits, and
    the emulated schedule equals the oracle on the slice."""
    rng = np.random.default_rng(9)
    d = 12
    linear = 0
    for trial in range(8):
        ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
        out = [("x", d + 2)]
        ins = [("offset", d), ("dev", 2)]
        A = ll.Layout(ins, out, {"offset": [(c,) for c in ca], "dev": [(1 << d,), (2 << d,)]})
        B = ll.Layout(ins, out, {"offset": [(c,) for c in cb], "dev": [(1 << d,), (2 << d,)]})
        p = ll.ll_plan_convert(A, B, 4)
        t = p.describe()
        assert t["class"] == "CTA" and t["exec"] == "tile"
        linear += bool(t["tile"].get("linear_tile"))
        OA = O.layout_from_cols([("offset", d)], [("x", d)], ca)
        OB = O.layout_from_cols([("offset", d)], [("x", d)], cb)
        src = gen.random_bits(rng, 1 << d, 4)
        assert np.array_equal(p.simulate(src, 1 << d), O.convert(OA, OB, src))
    assert linear >= 4


@pytest.mark.parametrize("balance", ["0", "1"])
def test_linear_tile_run_choice_simulated(monkeypatch, balance):
    """Linear tiles under both run choices (LL_LINEAR_BALANCE): widest store runs, or the
    longest shorter run of the two sides.  The tile holds dst bits [0, cs) and the
    preimages of src bits [0, cl); the first cs - v lanes store consecutive dst bits.
    Emulated schedules of random R2 memory layouts equal the oracle."""
    monkeypatch.setenv("LL_LINEAR_BALANCE", balance)
    shorter = 0
    tiles = 0
    for w in (1, 2, 4, 8):
        rng = np.random.default_rng(700 + w)
        for d in (12, 14, 16):
            for _ in range(3):
                ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
                ins, out = [("offset", d)], [("x", d)]
                OA, OB = O.layout_from_cols(ins, out, ca), O.layout_from_cols(ins, out, cb)
                A = ll.Layout(ins, out, {"offset": [(c,) for c in ca]})
                B = ll.Layout(ins, out, {"offset": [(c,) for c in cb]})
                p = ll.ll_plan_convert(A, B, w)
                t = p.describe()
                if t["exec"] != "tile" or not t["tile"].get("linear_tile"):
                    continue
                tiles += 1
                T = t["tile"]
                v = T["vst"]
                cs = T["st_run_bits"]
                assert v + 2 <= cs <= v + 5
                lanes = T["st_bit"][T["R"]:T["R"] + 5]
                assert lanes[:cs - v] == list(range(v, cs))
                shorter += cs < v + 5
                src = gen.random_bits(rng, 1 << d, w)
                assert np.array_equal(p.simulate(src, 1 << d), O.convert(OA, OB, src)), (w, d)
    assert tiles >= 20
    if balance == "0":
        assert shorter == 0
    else:
        assert shorter > 0


def test_linear_tiles_default_exchange(monkeypatch):
    """Without LL_PIPE / LL_MIN_BLOCKS, linear-tile plans (random R2 memory layouts) take
    the unpipelined smem exchange with two CTAs per SM (register cap) and opaque thread
    bases (NOHOIST); config 3 keeps the plain kernel with 2 CTAs per SM (8 warps x 256 B
    per thread: the register cap that keeps all 16 loads of a thread in flight)."""
    monkeypatch.delenv("LL_MIN_BLOCKS", raising=False)
    monkeypatch.delenv("LL_NOHOIST", raising=False)
    monkeypatch.delenv("LL_PIPE", raising=False)
    A, B = (ll.Layout.from_spec(x) for x in W.c3(9))
    p = ll.ll_plan_convert(A, B, 2)
    assert p.describe()["tile"]["pipe"] is False and p.describe()["tile"]["min_blocks"] == 2
    assert "NOHOIST = false" in p.source()
    rng = np.random.default_rng(801)
    seen = 0
    for _ in range(6):
        d = 18
        ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
        ins, out = [("offset", d)], [("x", d)]
        t = ll.ll_plan_convert(ll.Layout(ins, out, {"offset": [(c,) for c in ca]}),
                               ll.Layout(ins, out, {"offset": [(c,) for c in cb]}), 4).describe()
        if t["exec"] == "tile" and t["tile"].get("linear_tile") and t["tile"]["xchg"] == "smem":
            assert t["tile"]["pipe"] is False and t["tile"]["min_blocks"] == 2
            seen += 1
    assert seen >= 1


def test_plan_opts_pipe_and_min_blocks():
    """ll_plan_opts.pipe / min_blocks reach the plan (describe) and the generated kernel
    (__launch_bounds__ minimum): auto = linear tiles unpipelined with two CTAs per SM;
    explicit values override; in-CTA smem plans of 8 warps x 256 B per thread ask for
    two CTAs per SM; other smem plans keep the plain kernel."""
    rng = np.random.default_rng(9)
    d = 16
    ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
    ins, out = [("offset", d)], [("x", d)]
    A = ll.Layout(ins, out, {"offset": [(c,) for c in ca]})
    B = ll.Layout(ins, out, {"offset": [(c,) for c in cb]})
    for w, mb_auto in ((2, 2), (4, 2)):
        p = ll.ll_plan_convert(A, B, w)
        t = p.describe()["tile"]
        assert t["linear_tile"] and t["pipe"] is False and t["min_blocks"] == mb_auto
        assert (", 2)" in p.source()) == (mb_auto == 2) and "NOHOIST = true" in p.source()
        assert ll.ll_plan_convert(A, B, w, pipe="on").describe()["tile"]["pipe"] is True
        t = ll.ll_plan_convert(A, B, w, pipe="off", min_blocks=-1).describe()["tile"]
        assert t["pipe"] is False and t["min_blocks"] == 0
        p = ll.ll_plan_convert(A, B, w, min_blocks=3)
        assert p.describe()["tile"]["min_blocks"] == 3 and ", 3) ll_tile_kernel" in p.source()
    Ac, Bc = (ll.Layout.from_spec(x) for x in W.c3(9))
    t = ll.ll_plan_convert(Ac, Bc, 2).describe()["tile"]
    assert t["pipe"] is False and t["min_blocks"] == 2     # 8 warps x 256 B per thread
    assert ll.ll_plan_convert(Ac, Bc, 2, min_blocks=-1).describe()["tile"]["min_blocks"] == 0
    t = ll.ll_plan_convert(Ac, Bc, 2, pipe="on").describe()["tile"]
    assert t["pipe"] is True and t["min_blocks"] == 0
    Ac, Bc = (ll.Layout.from_spec(x) for x in W.c5T(0, n=12))     # 128 B per thread: no cap
    assert ll.ll_plan_convert(Ac, Bc, 2).describe()["tile"]["min_blocks"] == 0


def test_opts_struct_matches_the_c_abi():
    """The Python mirror of ll_plan_opts has the C struct's size: ll_plan_opts_default
    (memset + defaults) writes exactly sizeof(ll_plan_opts) bytes of a guarded buffer."""
    n = ctypes.sizeof(ll._Opts)
    buf = (ctypes.c_ubyte * (n + 64))(*([0xAB] * (n + 64)))
    ll._lib.ll_plan_opts_default(ctypes.cast(buf, ctypes.POINTER(ll._Opts)))
    assert all(b == 0xAB for b in buf[n:])
    assert any(b != 0xAB for b in buf[n - 8:n])        # the last fields were written
    o = ll._Opts.from_buffer(buf)
    assert o.force_class == -1 and o.max_vec_bytes == 16 and o.pipe == 0 and o.min_blocks == 0


def test_planned_wavefronts_equal_ncu_sass_counts():
    """the planner's predicted shared-memory wavefronts per tile (Lemma 9.4
    model) times the tiles of the launch equal the SASS-attributed wavefronts
    ncu counted on the B200 for the same plans (committed capture
    profiles/r01_smem_sass_wavefronts.json, tools/jobs/job59.sh), for every smem-exchange
    kernel captured — and both equal the conflict-free ideal (bytes / 128)."""
    import json
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                        "r01_smem_sass_wavefronts.json")
    m = json.load(open(path))["cases"]
    cases = {"c3": (W.c3(14), 2, {}), "c3b": (W.c3b(14), 2, {"force_class": "SMEM"}), "c5T": (W.c5T(0, n=15), 2, {}),
             "n1": (W.n1_preshuffle(14, 14), 2, {}), "c1bsmem": (W.c1_batched(20), 4, {"force_class": "SMEM"}),
             "c2smem": (W.c2(16), 2, {"force_class": "SMEM"}), "c3f": (W.c3(14), 2, {"sigma": "faithful"})}
    assert sorted(cases) == sorted(m)
    for k, ((sa, sb), w, o) in cases.items():
        t = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w, **o).describe()["tile"]
        nt = t["ctas"]
        assert t["wavefronts_st"] * nt == m[k]["st"]["sass_wavefronts"] == m[k]["st"]["ideal_wavefronts"], k
        assert t["wavefronts_ld"] * nt == m[k]["ld"]["sass_wavefronts"] == m[k]["ld"]["ideal_wavefronts"], k


def test_ncu_dram_traffic_within_algorithmic_bytes():
    """DRAM read + write bytes per launch that ncu measured for every bench
    kernel (profiles/ncu_traffic.json, the `roofline.traffic` source) stay within 1.05x of
    the algorithmic bytes (each element read once and written once; gather: src + idx +
    dst; reduce: src + dst) — no wasted re-reads."""
    import json
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_traffic.json")
    t = json.load(open(path))
    GiB, MiB = 1 << 30, 1 << 20
    algo = {"c2_shuffle": 4 * GiB, "c3": 2 * GiB, "c3b": 2 * GiB, "c1b": 2 * GiB, "c5T": 4 * GiB,
            "n1": GiB, "n2": GiB, "c5_peer_one_rank": 512 * MiB,   # P = 8: one rank moves 256 MiB in + out
            "gather_mma": 192 * MiB, "gather_blocked": 192 * MiB,
            "reduce_mma": 64 * MiB + MiB // 2, "reduce_blocked": 64 * MiB + MiB // 2}
    for k, a in algo.items():
        assert t[k] <= 1.05 * a, (k, t[k], a)


@pytest.mark.parametrize("n_zero", [1, 3, 5, 6, 7, 8])
def test_broadcast_sweep_specialised_and_simulated(n_zero):
    """Broadcast targets with up to 8 zero columns stay on the specialised
    tile kernel (replica stores: 16 unrolled, the rest looped) — never the generic
    kernel — and the simulated schedule equals the oracle's conversion."""
    rng = np.random.default_rng(500 + n_zero)
    for case in range(12):
        sa, sb = gen.random_broadcast_pair(rng, n_zero, batch_bits=2)
        w = [1, 2, 4, 8][case % 4]
        d = _sim_check(sa, sb, w, case)
        assert d["exec"] == "tile", d
        t = d["tile"]
        low = len(t["bcast_U"]) - t["n"] if t["bcast_store"] else 0
        assert len(t["rep_bits"]) + low == n_zero


def test_broadcast_probe_never_generic():
    """300 random distributed -> broadcast pairs (5-8 zero columns, batched): the
    planner picks the generic kernel for none of them."""
    rng = np.random.default_rng(300)
    for _ in range(300):
        sa, sb = gen.random_broadcast_pair(rng, int(rng.integers(5, 9)), ki=7, kj=7, batch_bits=10)
        p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 4)
        assert p.describe()["exec"] == "tile"


@pytest.mark.parametrize("shape", ["32x32b", "16x64b", "16x128b", "16x256b"])
@pytest.mark.parametrize("N", [8, 64, 256])
def test_tmem_family_matches_oracle(shape, N):
    """ll_layout_tmem (product) == O.tmem_ld (oracle, pinned to the CUTLASS SM100
    TMEM_LOAD traits) column by column."""
    L = ll.ll_layout_tmem(shape, 128, N)
    assert L.cols() == O.tmem_ld(shape, 128, N).cols


def test_tmem_family_errors():
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_layout_tmem("16x32b", 128, 64)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_layout_tmem("16x256b", 64, 64)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_layout_tmem("16x256b", 128, 4)


@pytest.mark.parametrize("shape", ["32x32b", "16x64b", "16x128b", "16x256b"])
def test_n2_tmem_epilogue_simulated(shape):
    """TMEM fragment -> coalesced blocked epilogue layout: the planner's class equals
    the oracle's and the simulated schedule equals the oracle's conversion."""
    sa, sb = W.n2_tmem(shape, nb=1)
    A, OA = both(sa)
    B, OB = both(sb)
    assert ll.ll_plan_convert(A, B, 4).cls == O.classify(OA, OB)
    d = _sim_check(sa, sb, 4, 3)
    assert d["exec"] == "tile"


@pytest.mark.parametrize("bits", [8, 16])
def test_n2_acc_to_lhs_simulated(bits):
    sa, sb = W.n2_acc_to_lhs(bits, nb=2)
    A, OA = both(sa)
    B, OB = both(sb)
    p = ll.ll_plan_convert(A, B, bits // 8)
    assert p.cls == ("NOOP" if bits == 16 else "SHUFFLE")
    if bits == 8:
        # default (coalesced HBM vectors of 16 fp8) and the layouts' own registers
        # (faithful σ).  The executed exchange is smem in both: a 32-bit shuffle unit
        # holds (j0, i3) in A but (j0, j1) in B (reading R-V)
        for seed, opts in ((4, {}), (5, {"sigma": "faithful"})):
            d = _sim_check(sa, sb, 1, seed, **opts)
            assert d["exec"] == "tile"


def test_permuted_subword_shuffles_simulated():
    """Sub-word shuffles whose 32-bit unit is not common at the lowest registers (reading
    R-V): random SHUFFLE-class pairs with 1- and 2-byte elements; the plans that take the
    element-permuted shuffle (plan_shuffle_eperm) reproduce the oracle's conversion in
    the host emulation, and some do."""
    rng = np.random.default_rng(31)
    out = [("i", 5), ("j", 5)]
    seen = 0
    for case in range(400):
        r = int(rng.integers(3, 6))
        hw = [("reg", r), ("lane", 5), ("warp", 10 - r - 5)]
        sa = gen.random_distributed(rng, out, hw)
        sb = gen.random_distributed(rng, out, hw)
        for w in (1, 2):
            A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
            d = ll.ll_plan_convert(A, B, w).describe()
            if d.get("tile", {}).get("element_permutes"):
                seen += 1
                dd = _sim_check(sa, sb, w, case)
                assert dd["class"] == "SHUFFLE"
    assert seen >= 5, seen


@pytest.mark.parametrize("n_zero", [1, 3, 6])
def test_broadcast_cta_class_simulated(n_zero):
    """Broadcast targets whose block bits are permuted (CTA class): the data bits run as a
    CTA-tiled permutation with replica stores — no XOR-copy or generic kernel — and the
    simulated schedule equals the oracle's conversion."""
    import os
    rng = np.random.default_rng(700 + n_zero)
    old = os.environ.get("LL_BCAST_CTA")
    try:
        for mode in ("1", None):      # CTA-tiled broadcast first; the default order
            if mode:
                os.environ["LL_BCAST_CTA"] = mode
            else:
                os.environ.pop("LL_BCAST_CTA", None)
            for case in range(10):
                sa, sb = gen.random_broadcast_pair(rng, n_zero, batch_bits=4, permute_batch=True)
                w = [1, 2, 4, 8][case % 4]
                d = _sim_check(sa, sb, w, case)
                assert d["exec"] == "tile", d
                if mode == "1":
                    assert "ld_xcol" not in d["tile"], d
    finally:
        if old is None:
            os.environ.pop("LL_BCAST_CTA", None)
        else:
            os.environ["LL_BCAST_CTA"] = old


def test_convert_pointer_checks_before_launch():
    """ll_convert validates its pointers before touching the GPU: 16-byte alignment
    (LL_ERR_MISALIGNED) and src / dst overlap for non-NOOP plans (LL_ERR_ALIAS) — raw
    addresses, nothing is dereferenced."""
    A, B = ll.Layout.from_spec(W.C1_A), ll.Layout.from_spec(W.C1_B)
    p = ll.ll_plan_convert(A, B, 4)
    base = 1 << 32
    with pytest.raises(ll.LLError, match="MISALIGNED"):
        ll.ll_convert(base + 4, base + 4096, p, stream=0)
    with pytest.raises(ll.LLError, match="ALIAS"):
        ll.ll_convert(base, base + 512, p, stream=0)      # 1 KiB buffers overlapping by half


def test_noop_partial_overlap_refused():
    """NOOP plans (A = B) run in place when src == dst and as a streaming copy kernel
    otherwise; partially overlapping buffers are refused (LL_ERR_ALIAS) before any
    launch — raw addresses, nothing is dereferenced."""
    A = ll.Layout.from_spec(W.C1_A)
    p = ll.ll_plan_convert(A, A, 4)
    assert p.cls == "NOOP"
    base = 1 << 32
    with pytest.raises(ll.LLError, match="ALIAS"):
        ll.ll_convert(base, base + 512, p, stream=0)      # 1 KiB buffers overlapping by half


def test_round2_kernel_shape_defaults():
    """Measured defaults: folded small tiles run 8 warps x 64 B per
    thread; shuffle / smem tiles of 256 B per thread with <= 8 warps carry the 2-CTA
    register hint (config 2, config 3); the CTA-class transpose (128 B per thread) and
    config 2's own 4-warp shuffle keep their shapes."""
    def tile(spec, w, **o):
        A, B = (ll.Layout.from_spec(x) for x in spec)
        return ll.ll_plan_convert(A, B, w, **o).describe()["tile"]
    t = tile(W.c2(4), 2)
    assert t["xchg"] == "shuffle" and t["threads"] == 128 and t["min_blocks"] == 2
    t = tile(W.c3(4), 2)
    assert t["xchg"] == "smem" and t["threads"] == 256 and t["min_blocks"] == 2
    t = tile(W.c1_batched(12), 4)
    assert t["threads"] == 256 and t["R"] == 4          # 16 KiB folded tile, 64 B per thread
    assert tile(W.c1_batched(12), 4, thread_bytes=256)["threads"] == 64
    t = tile(W.c5T(0, n=12), 2)
    assert t["min_blocks"] == 0
