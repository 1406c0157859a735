"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by
element, bit-exact (movement is integer work).  Needs a B200 (-m gpu)."""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen
from tests._util import empty_device, from_device, to_device

pytestmark = pytest.mark.gpu

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def both(spec):
    return ll.Layout.from_spec(spec), O.Layout(*W.spec_to_bases(spec))


def run_convert(sa, sb, w, seed, **opts):
    A, OA = both(sa)
    B, OB = both(sb)
    rng = np.random.default_rng(seed)
    T = gen.random_bits(rng, 1 << OA.d_out, w)
    src = O.pack(OA, T)
    plan = ll.ll_plan_convert(A, B, w, **opts)
    d_src = to_device(src)
    d_dst = empty_device(1 << OB.d_in, w)
    ll.ll_convert(d_src, d_dst, plan)
    import torch
    torch.cuda.synchronize()
    got = from_device(d_dst, w)
    ref = O.convert(OA, OB, src)
    return got, ref, plan


CASES = [
    ("c1", (W.C1_A, W.C1_B), 4),
    ("c1_batch", W.c1_batched(6), 4),
    ("c2", W.c2(3), 2),
    ("c3", W.c3(2), 2),
    ("c3b", W.c3b(2), 2),
]


@pytest.mark.parametrize("name,specs,w", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("force", [None, "SMEM"])
def test_configs_small_bitexact(name, specs, w, force):
    got, ref, plan = run_convert(specs[0], specs[1], w, 1001, force_class=force)
    assert plan.describe()["exec"] == "tile"
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("name,specs,w", CASES[:4], ids=[c[0] for c in CASES[:4]])
def test_configs_faithful_sigma(name, specs, w):
    got, ref, plan = run_convert(specs[0], specs[1], w, 7, sigma="faithful")
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_random_distributed_bijective(w):
    rng = np.random.default_rng(100 + w)
    out = [("b", 3), ("i", 5), ("j", 5)]
    hw = [("reg", 2), ("lane", 5), ("warp", 3)]
    for case in range(6):
        sa = gen.random_distributed(rng, out[1:], hw)
        sb = gen.random_distributed(rng, out[1:], hw)
        # batch bits as block dims, identical in A and B
        sa = {"out": out, "in": sa["in"] + [("block", ["b0", "b1", "b2"])]}
        sb = {"out": out, "in": sb["in"] + [("block", ["b0", "b1", "b2"])]}
        got, ref, plan = run_convert(sa, sb, w, case)
        assert np.array_equal(got, ref), (case, plan.describe()["class"])


def test_random_cta_class():
    rng = np.random.default_rng(5)
    out = [("i", 6), ("j", 6)]
    for case in range(6):
        cols_a = rng.permutation(12)
        cols_b = rng.permutation(12)
        name = lambda k: f"j{k}" if k < 6 else f"i{k - 6}"
        sa = {"out": out, "in": [("offset", [name(k) for k in cols_a])]}
        sb = {"out": out, "in": [("offset", [name(k) for k in cols_b])]}
        got, ref, plan = run_convert(sa, sb, 2, case)
        assert np.array_equal(got, ref), plan.describe()["class"]


def test_broadcast_generic():
    rng = np.random.default_rng(9)
    out = [("i", 3), ("j", 4)]
    hw = [("reg", 2), ("lane", 5), ("warp", 1)]
    for case in range(5):
        sa = gen.random_distributed(rng, out, hw, zero_ok=["reg"])
        sb = gen.random_distributed(rng, out, hw, zero_ok=["lane"])
        got, ref, plan = run_convert(sa, sb, 4, case)
        assert np.array_equal(got, ref)


def test_memory_swizzle_generic():
    """Def 4.14 memory layouts with 2-bit columns (R2): non-permutation pull map."""
    rng = np.random.default_rng(21)
    for case in range(5):
        d = 10
        ca = gen.random_memory_cols(rng, d)
        cb = gen.random_memory_cols(rng, d)
        out = [("x", d)]
        OA = O.layout_from_cols([("offset", d)], out, ca)
        OB = O.layout_from_cols([("offset", d)], out, cb)
        A = ll.Layout([("offset", d)], out, {"offset": [(c,) for c in ca]})
        B = ll.Layout([("offset", d)], out, {"offset": [(c,) for c in cb]})
        src = gen.random_bits(rng, 1 << d, 4)
        plan = ll.ll_plan_convert(A, B, 4)
        d_src, d_dst = to_device(src), empty_device(1 << d, 4)
        ll.ll_convert(d_src, d_dst, plan)
        assert np.array_equal(from_device(d_dst, 4), O.convert(OA, OB, src))


def test_noop_memcpy():
    A, OA = both(W.C1_A)
    plan = ll.ll_plan_convert(A, A, 4)
    assert plan.cls == "NOOP"
    src = gen.random_bits(np.random.default_rng(0), 256, 4)
    d_src, d_dst = to_device(src), empty_device(256, 4)
    ll.ll_convert(d_src, d_dst, plan)
    assert np.array_equal(from_device(d_dst, 4), src)


@pytest.mark.parametrize("d", [0, 1, 3, 4, 9, 12, 21])
@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_noop_copy_kernel_sizes(d, w):
    """NOOP plans with dst != src run ll_copy_kernel (32 KiB per CTA): buffers from one
    element (a bytewise tail below 16 bytes) through partial and many CTA tiles equal
    the input; src == dst is accepted and leaves the buffer unchanged."""
    out = [("x", d)]
    A = ll.Layout([("offset", d)], out, {"offset": [(1 << k,) for k in range(d)]})
    plan = ll.ll_plan_convert(A, A, w)
    assert plan.cls == "NOOP"
    src = gen.random_bits(np.random.default_rng(d * 8 + w), 1 << d, w)
    d_src, d_dst = to_device(src), empty_device(1 << d, w)
    ll.ll_convert(d_src, d_dst, plan)
    assert np.array_equal(from_device(d_dst, w), src)
    ll.ll_convert(d_dst, d_dst, plan)
    assert np.array_equal(from_device(d_dst, w), src)


def _full_size_every_element(sa, sb, w, nsample_seed):
    _full_size_every_element_opts(sa, sb, w, nsample_seed)


def _full_size_every_element_opts(sa, sb, w, nsample_seed, **opts):
    """Full-size conversion in bench.py's launch configuration (the default plan):
    src hash-filled (src[h] = H(A(h)), workloads/hashfill.py), then EVERY dst element
    compared on the device with the closed form H(B(h)) (O5), and 2^20 sampled outputs
    additionally against the oracle's pull map A^+(B(h)) one by one."""
    import torch
    from workloads import hashfill as H
    A, OA = both(sa)
    B, OB = both(sb)
    plan = ll.ll_plan_convert(A, B, w, **opts)
    src = H.fill(sa, w, nsample_seed)
    n = src.numel()
    dst = torch.empty_like(src)
    ll.ll_convert(src, dst, plan)
    torch.cuda.synchronize()
    assert H.check(sb, w, nsample_seed, dst) == 0
    rng = np.random.default_rng(nsample_seed)
    hs = np.concatenate([rng.integers(0, n, size=1 << 20), np.arange(4096), n - 1 - np.arange(4096)]).astype(np.uint64)
    hsrc = O.apply_inverse_all(OA, O.apply_all(OB, hs)).astype(np.int64)
    got = dst[torch.from_numpy(hs.astype(np.int64)).cuda()].cpu().numpy()
    want = src[torch.from_numpy(hsrc).cuda()].cpu().numpy()
    assert np.array_equal(got, want)
    del src, dst
    torch.cuda.empty_cache()


def test_config2_full_size():
    """BASELINE config 2 at full size (65536 tiles, 2^30 bf16 elements)."""
    _full_size_every_element(*W.c2(16), 2, 1002)


def test_config3_full_size():
    """BASELINE config 3 at full size (16384 tiles, 2^29 fp16 elements)."""
    _full_size_every_element(*W.c3(14), 2, 1003)


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("sigma", ["coalesced", "faithful"])
@pytest.mark.parametrize("k_bits", [4, 5, 6])
@pytest.mark.parametrize("exchange", ["SHUFFLE", "SMEM", "LDG"])
def test_gather_bitexact(family, sigma, k_bits, exchange):
    """O10: gather via shuffles or via shared memory (the P:519 crossover)
    vs the oracle (take_along_axis), for the config-4 tiles [128, K], K = 16 / 32 / 64
    (the survey's K sweep)."""
    rng = np.random.default_rng(1004)
    spec = W.c4("gather", family, n_i=9, n_j=7, k_bits=k_bits)
    L, OL = both(spec)
    n = 1 << OL.d_in
    T = gen.random_bits(rng, n, 4)
    Ti = rng.integers(-1000, 1000, size=n).astype(np.int32)   # masked to [0, K) (G16)
    src, idx = O.pack(OL, T), O.pack(OL, Ti)
    ref = O.gather(OL, 1, src, idx)
    # SHUFFLE / SMEM: forced exchange, TMA-staged when coalesced (pipe = bulk); LDG: the
    # default plan (automatic exchange, direct global loads)
    if exchange == "LDG":
        plan = ll.ll_plan_gather(L, 1, 4, sigma=sigma)
    else:
        plan = ll.ll_plan_gather(L, 1, 4, sigma=sigma, force_class=exchange, pipe="bulk")
    d = plan.describe()
    if exchange != "LDG":
        assert d["exchange"] == exchange.lower()
        assert d["tma"] == (sigma == "coalesced")
    else:
        assert not d["tma"]
    d_dst = empty_device(n, 4)
    ll.ll_gather(to_device(src), to_device(idx.view(np.uint32)), d_dst, plan)
    assert np.array_equal(from_device(d_dst, 4), ref)


@pytest.mark.parametrize("w", [2, 1])
@pytest.mark.parametrize("exchange", ["SHUFFLE", "SMEM"])
def test_gather_narrow_elements(w, exchange):
    rng = np.random.default_rng(1009)
    spec = W.c4("gather", "mma", n_i=8, n_j=6, k_bits=5)
    L, OL = both(spec)
    n = 1 << OL.d_in
    T = gen.random_bits(rng, n, w)
    Ti = rng.integers(0, 32, size=n).astype(np.int32)
    src, idx = O.pack(OL, T), O.pack(OL, Ti)
    plan = ll.ll_plan_gather(L, 1, w, force_class=exchange)
    d_dst = empty_device(n, w)
    ll.ll_gather(to_device(src), to_device(idx.view(np.uint32)), d_dst, plan)
    assert np.array_equal(from_device(d_dst, w), O.gather(OL, 1, src, idx))


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("sigma", ["coalesced", "coalesced-tma", "faithful"])
def test_reduce_tolerance_and_fixed_order(family, sigma):
    """O11: ≤ 1e-6 relative vs fp64, and bit-exact vs the fixed-order fp32 replica on
    L itself (reading R-reduce: logical axis-bit order), for every kernel layout σ and
    load path — the bits do not depend on plan options."""
    import torch
    rng = np.random.default_rng(1005)
    spec = W.c4("reduce", family, n_i=9, n_j=9)
    L, OL = both(spec)
    n = 1 << OL.d_in
    T = rng.random(n, dtype=np.float32)
    src = O.pack(OL, T)
    # "coalesced" loads directly (the default for reduces without a warp step),
    # "coalesced-tma" stages tiles with cp.async.bulk (TMA, opts.pipe = bulk)
    plan = ll.ll_plan_reduce(L, 1, sigma=sigma.split("-")[0], pipe="bulk" if sigma == "coalesced-tma" else "auto")
    assert plan.describe()["tma"] == (sigma == "coalesced-tma")
    out = torch.empty(plan.out_elems(), dtype=torch.float32, device="cuda")
    ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan)
    got = out.cpu().numpy()
    ref = O.reduce_ref_fp64(OL, 1, src)
    assert np.all(np.abs(got - ref) <= 1e-6 * np.abs(ref))
    rep = O.reduce_fixed_order_fp32(OL, 1, src)
    assert np.array_equal(got.view(np.uint32), rep.view(np.uint32))


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("sigma", ["coalesced", "faithful"])
@pytest.mark.parametrize("op", ["max", "min"])
def test_reduce_max_min_bitexact(family, sigma, op):
    """max / min reductions (ll_plan_opts.reduce_op) along axis 1 inside [128,128]
    tiles: exact, so bit-equal to the oracle's fp64 reference."""
    import torch
    rng = np.random.default_rng(1006)
    L, OL = both(W.c4("reduce", family, n_i=9, n_j=9))
    n = 1 << OL.d_in
    T = (rng.random(n, dtype=np.float32) - 0.5).astype(np.float32)
    src = O.pack(OL, T)
    plan = ll.ll_plan_reduce(L, 1, sigma=sigma, reduce_op=op)
    assert plan.describe()["op"] == op
    out = torch.empty(plan.out_elems(), dtype=torch.float32, device="cuda")
    ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan)
    ref = O.reduce_ref_fp64(OL, 1, src, op).astype(np.float32)
    assert np.array_equal(out.cpu().numpy().view(np.uint32), ref.view(np.uint32))


def test_reduce_broadcast_dedup_gpu():
    """a layout with zero columns (duplicated lanes and registers) reduces each
    logical element once; one write per output."""
    import torch
    OL = O.blocked([8, 16], [1, 2], [4, 8], [4, 1], [1, 0])
    spec = {"out": [("d0", 3), ("d1", 4)], "in": []}
    L = ll.Layout(OL.in_dims, OL.out_dims, OL.bases)
    rng = np.random.default_rng(3)
    T = rng.random(128, dtype=np.float32)
    src = O.pack(OL, T)
    plan = ll.ll_plan_reduce(L, 1, sigma="faithful")
    out = torch.full((plan.out_elems(),), -1.0, dtype=torch.float32, device="cuda")
    ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan)
    got = out.cpu().numpy()
    rep = O.reduce_fixed_order_fp32(OL, 1, src)
    assert np.array_equal(got.view(np.uint32), rep.view(np.uint32))


def test_exhaustive_fig1_sample_gpu():
    """E1 (sampled on GPU): random bijective relabelings B of Fig. 1's 2^8 space
    against Fig. 1 A, and a 7-bit space where A and B each carry a broadcast column;
    every plan (tile kernel or generic kernel) bit-exact against the oracle, and the
    planner's class equal to the oracle's existential class (O7)."""
    import torch
    rng = np.random.default_rng(4040)
    A, OA = both(W.C1_A)
    hw = [("reg", 2), ("lane", 5), ("warp", 1)]
    T = gen.random_bits(rng, 256, 4)
    src = O.pack(OA, T)
    d_src = to_device(src)
    for case in range(60):
        sb = gen.random_distributed(rng, W.C1_OUT, hw)
        B, OB = both(sb)
        plan = ll.ll_plan_convert(A, B, 4)
        assert plan.cls == O.classify(OA, OB)
        d_dst = empty_device(256, 4)
        ll.ll_convert(d_src, d_dst, plan)
        assert np.array_equal(from_device(d_dst, 4), O.pack(OB, T)), (case, plan.describe()["exec"])
    out7 = [("i", 3), ("j", 4)]
    T7 = gen.random_bits(rng, 128, 4)
    for case in range(30):
        sa = gen.random_distributed(rng, out7, hw, zero_ok=["reg"])
        sb = gen.random_distributed(rng, out7, hw, zero_ok=["lane"])
        A7, OA7 = both(sa)
        B7, OB7 = both(sb)
        plan = ll.ll_plan_convert(A7, B7, 4)
        assert plan.cls == O.classify(OA7, OB7)
        d_dst = empty_device(256, 4)
        ll.ll_convert(to_device(O.pack(OA7, T7)), d_dst, plan)
        assert np.array_equal(from_device(d_dst, 4), O.pack(OB7, T7))


@pytest.mark.parametrize("want", ["REGPERM", "SHUFFLE"])
def test_class_kernels_faithful_gpu(want):
    """Register permutation and warp shuffles executed on the
    layouts' own hardware (faithful σ), so the executed exchange is the paper's class;
    random pairs built by permuting register bits (REGPERM) or register+lane bits
    (SHUFFLE) of a random distributed layout; 4-byte and 2-byte elements."""
    rng = np.random.default_rng(606 if want == "REGPERM" else 607)
    out = [("b", 4), ("i", 5), ("j", 5)]
    hw = [("reg", 3), ("lane", 5), ("warp", 2)]
    done = 0
    for case in range(60):
        sa = gen.random_distributed(rng, out[1:], hw)
        ins = dict(sa["in"])
        if want == "REGPERM":
            regs = list(ins["reg"])
            rng.shuffle(regs)
            sb_in = [("reg", regs), ("lane", ins["lane"]), ("warp", ins["warp"])]
        else:
            pool = list(ins["reg"]) + list(ins["lane"])
            rng.shuffle(pool)
            sb_in = [("reg", pool[:3]), ("lane", pool[3:]), ("warp", ins["warp"])]
        blk = [("block", ["b0", "b1", "b2", "b3"])]
        sa = {"out": out, "in": sa["in"] + blk}
        sb = {"out": out, "in": sb_in + blk}
        OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
        if O.classify(OA, OB) != want:
            continue
        for w in (4, 2):
            got, ref, plan = run_convert(sa, sb, w, case, sigma="faithful")
            d = plan.describe()
            assert d["class"] == want
            if w == 4:
                assert d["tile"]["xchg"] == {"REGPERM": "regperm", "SHUFFLE": "shuffle"}[want]
            assert np.array_equal(got, ref), (case, w)
        done += 1
        if done == 8:
            break
    assert done >= 5


@pytest.mark.parametrize("which", ["n1", "n2"])
def test_next_rows_n1_n2_bitexact(which):
    """§8(f) N1 (HBM pre-shuffle of a bf16 weight into mma rhs fragment order)
    and N2 (tcgen05 TMEM 32x32b fragment -> coalesced blocked epilogue layout)."""
    if which == "n1":
        (sa, sb), w = W.n1_preshuffle(9, 8), 2
    else:
        (sa, sb), w = W.n2_tmem_epilogue(3), 4
    got, ref, plan = run_convert(sa, sb, w, 77)
    assert plan.describe()["exec"] == "tile"
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("which", ["tmem_32x32b", "tmem_16x64b", "tmem_16x128b", "tmem_16x256b",
                                   "acc_lhs_bf16", "acc_lhs_fp8"])
@pytest.mark.parametrize("sigma", ["coalesced", "faithful"])
def test_n2_families_bitexact(which, sigma):
    """§8(f) N2: every tcgen05.ld fragment shape (ll_layout_tmem; CUTLASS-pinned oracle
    tables) -> coalesced blocked epilogue layout, and the chained-GEMM wgmma accumulator
    -> register-A operand conversions (bf16: NOOP; fp8: SHUFFLE class) — small batches
    against the oracle's conversion."""
    if which.startswith("tmem"):
        (sa, sb), w = W.n2_tmem(which[5:], 3), 4
    else:
        bits = 16 if which.endswith("bf16") else 8
        (sa, sb), w = W.n2_acc_to_lhs(bits, 4), bits // 8
    got, ref, plan = run_convert(sa, sb, w, 78, sigma=sigma)
    assert plan.describe()["exec"] in ("tile", "noop")
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("which", ["n1", "tmem_16x64b", "tmem_16x128b", "tmem_16x256b", "acc_lhs_fp8"])
def test_next_rows_full_size_every_element(which):
    """N1 / N2 at the bench's sizes (1-2 GiB): every element against H(B(h))."""
    if which == "n1":
        (sa, sb), w = W.n1_preshuffle(15, 15), 2
    elif which.startswith("tmem"):
        (sa, sb), w = W.n2_tmem(which[5:], 14), 4
    else:
        (sa, sb), w = W.n2_acc_to_lhs(8, 18), 1
    _full_size_every_element(sa, sb, w, 4242)


def test_broadcast_tile_kernels_gpu():
    """Broadcast (zero-column) layouts through the specialised kernels (rule (2),
    P:362): bit-exact, and at least some plans execute as tile kernels."""
    rng = np.random.default_rng(55)
    opts_z = [["reg", "lane"], ["lane", "warp"], ["reg", "warp"]]
    tiles = 0
    for case in range(24):
        out = [("i", 4), ("j", 4)]
        hw = [("reg", 3), ("lane", 5), ("warp", 2)]
        sa = gen.random_distributed(rng, out, hw, zero_ok=opts_z[case % 3])
        sb = gen.random_distributed(rng, out, hw, zero_ok=opts_z[(case // 3) % 3])
        got, ref, plan = run_convert(sa, sb, [2, 4][case % 2], case)
        assert np.array_equal(got, ref), plan.describe()
        tiles += plan.describe()["exec"] == "tile"
    assert tiles >= 8


@pytest.mark.parametrize("n_streams,dev_bytes", [(2, 1 << 20), (3, (1 << 20) + 48), (4, 3 << 20)])
def test_convert_host_pipeline(n_streams, dev_bytes):
    """ll_convert_host: pinned host src -> chunked H2D / kernel / D2H over 2-4 streams
    (device scratch split into aligned slots, also for sizes not divisible by the
    stream count) -> pinned host dst, equal to the oracle."""
    import torch
    sa, sb = W.c2(6)
    A, OA = both(sa)
    B, OB = both(sb)
    plan = ll.ll_plan_convert(A, B, 2)
    rng = np.random.default_rng(8)
    src = O.pack(OA, gen.random_bits(rng, 1 << OA.d_out, 2))
    h_src = torch.from_numpy(src.view(np.int16).copy()).pin_memory()
    h_dst = torch.zeros_like(h_src).pin_memory()
    dev = torch.empty(dev_bytes, dtype=torch.uint8, device="cuda")    # forces several chunks
    streams = [torch.cuda.Stream() for _ in range(n_streams)]
    ll.ll_convert_host(h_src, h_dst, dev, plan, streams)
    torch.cuda.synchronize()
    assert np.array_equal(h_dst.numpy().view(np.uint16), O.convert(OA, OB, src))


# ---------------------------------------------------------------- N3: Table 4 families
TABLE4_SHAPES = [(128, 16), (128, 128), (32, 128), (32, 32), (16, 16)]


def _table4_layout(family, shape, rng):
    """(oracle layout, product layout) of one Table 4 family on `shape`,
    4 warps.  Sliced<F> is F on [a, b] times one extra register bit on a third
    dim, sliced away (Prop 4.8): a broadcast register (zero column)."""
    a, b = shape
    if family == "blocked":
        args = ([a, b], [1, 4], [8, 4], [4, 1], [1, 0])
        return O.blocked(*args), ll.ll_layout_blocked(*args)
    if family == "mma":
        return O.mma_acc([a, b], 4), ll.ll_layout_mma_acc(a, b, 4)
    if family == "mma_input":
        return O.mma_operand(False, (a, b), 16, 4, 1), ll.ll_layout_mma_operand(0, a, b, 16, 4, 1)
    if family.startswith("sliced_"):
        OP, _ = _table4_layout(family[len("sliced_"):], shape, rng)
        # parent over [a, b, 2]: the extra register bit hits the new dim, then slice it
        out3 = list(OP.out_dims) + [("d2", 1)]
        bases = {n: [tuple(v) + (0,) for v in OP.bases[n]] for n, _ in OP.in_dims}
        bases["reg"] = bases["reg"] + [(0, 0, 1)]
        in3 = [(n, nb + (1 if n == "reg" else 0)) for n, nb in OP.in_dims]
        parent = O.Layout(in3, out3, bases)
        OS = O.sliced(parent, 2)
        return OS, ll.Layout(OS.in_dims, OS.out_dims, OS.bases)
    # custom: a random distributed layout with broadcast lanes / registers
    out = [("r", a.bit_length() - 1), ("c", b.bit_length() - 1)]
    d = sum(x for _, x in out)
    nreg = max(1, d - 7 + 2)
    spec = gen.random_distributed(rng, out, [("reg", nreg), ("lane", 5), ("warp", 2)], zero_ok=["reg", "lane", "warp"])
    OL = O.Layout(*W.spec_to_bases(spec))
    return OL, ll.Layout(OL.in_dims, OL.out_dims, OL.bases)


@pytest.mark.parametrize("family", ["blocked", "mma", "mma_input", "sliced_blocked", "sliced_mma",
                                    "sliced_mma_input", "custom"])
def test_table4_reduce_families(family):
    """§8(f) N3: reductions (tl.sum) along either dim over every Table 4 layout family on
    the Table 4 shapes (5 shapes x 2 axes per family): ≤ 1e-6 relative vs
    fp64 and bit-exact vs the fixed-order replica (on L; no knowledge of the kernel's
    layout); broadcast copies counted once."""
    import torch
    rng = np.random.default_rng(4747)
    for shape in TABLE4_SHAPES:
        OL, L = _table4_layout(family, shape, rng)
        assert L.cols() == OL.cols
        T = rng.random(1 << OL.d_out, dtype=np.float32)
        src = O.pack(OL, T)
        for axis in (1, 0):
            plan = ll.ll_plan_reduce(L, axis)
            out = torch.full((plan.out_elems(),), -1.0, dtype=torch.float32, device="cuda")
            ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan)
            got = out.cpu().numpy()
            ref = T.astype(np.float64).reshape(shape).sum(axis=axis)
            assert np.all(np.abs(got - ref) <= 1e-6 * np.abs(ref)), (family, shape, axis)
            for sigma in ("coalesced", "faithful", "bulk"):
                if sigma != "coalesced":
                    plan = (ll.ll_plan_reduce(L, axis, sigma="faithful") if sigma == "faithful" else
                            ll.ll_plan_reduce(L, axis, pipe="bulk"))
                    out.fill_(-1.0)
                    ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan)
                    got = out.cpu().numpy()
                rep = O.reduce_fixed_order_fp32(OL, axis, src)
                assert np.array_equal(got.view(np.uint32), rep.view(np.uint32)), (family, shape, axis, sigma)


def test_swizzled_memory_layout_gpu():
    """Row-major -> Def 4.11 mma-swizzled memory layout of a 1024 x 1024 bf16 matrix
    (vec 8, per_phase 1, max_phase 8 — the 128-byte swizzle pattern) on the XOR-column
    copy kernel: element (i, j) lands at i*2^10 + Def 4.11 offset."""
    import torch
    m = n = 10
    S = ll.ll_layout_mma_swizzle(m, n, 8, 1, 8)
    R = ll.Layout([("offset", m + n)], [("d0", m), ("d1", n)],
                  {"offset": [((1 << (k - n)) if k >= n else 0, (1 << k) if k < n else 0) for k in range(m + n)]})
    plan = ll.ll_plan_convert(R, S, 2)
    assert plan.describe()["exec"] == "tile"
    T = gen.random_bits(np.random.default_rng(12), 1 << (m + n), 2)
    d_dst = empty_device(1 << (m + n), 2)
    ll.ll_convert(to_device(T), d_dst, plan)
    got = from_device(d_dst, 2)
    i = np.arange(1 << m)[:, None]
    j = np.arange(1 << n)[None, :]
    off = (i << n) + ((((i // 1) % 8) ^ (j // 8)) * 8 ^ (j % 8))
    assert np.array_equal(got[off.reshape(-1)], T)


@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_swizzled_memory_layouts_in_vector_xor_gpu(w):
    """Def 4.11 swizzles whose XOR reaches below the 16-byte vector (vec * w < 16):
    the XOR-copy kernel loads whole aligned src vectors and permutes the elements in
    registers (in-vector XOR).  Both directions, every parameter set, 256 x 256, each
    element (i, j) found at i*2^8 + the Def 4.11 offset (oracle formula)."""
    m = n = 8
    R = ll.Layout([("offset", m + n)], [("d0", m), ("d1", n)],
                  {"offset": [((1 << (k - n)) if k >= n else 0, (1 << k) if k < n else 0) for k in range(m + n)]})
    rng = np.random.default_rng(40 + w)
    i = np.arange(1 << m)[:, None]
    j = np.arange(1 << n)[None, :]
    for vec, pp, mp in [(1, 1, 8), (2, 1, 8), (4, 2, 4), (1, 2, 8), (1, 1, 4), (8, 1, 8), (16, 1, 8)]:
        S = ll.ll_layout_mma_swizzle(m, n, vec, pp, mp)
        off = ((i << n) + np.vectorize(lambda a, b: O.mma_swizzle_offset(int(a), int(b), vec, pp, mp))(i, j)).reshape(-1)
        T = gen.random_bits(rng, 1 << (m + n), w)
        for A, B in ((R, S), (S, R)):
            plan = ll.ll_plan_convert(A, B, w)
            d = plan.describe()
            assert d["exec"] == "tile" and (1 << d["tile"]["vld"]) * min(w, 4) == 16, d["tile"]["vld"]
            src = T if A is R else _scatter(T, off)
            d_dst = empty_device(1 << (m + n), w)
            ll.ll_convert(to_device(src), d_dst, plan)
            got = from_device(d_dst, w)
            want = _scatter(T, off) if A is R else T
            assert np.array_equal(got, want), (vec, pp, mp, A is R)


def _scatter(T, off):
    out = np.empty_like(T)
    out[off] = T
    return out


@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_linear_tiles_random_memory_layouts_gpu(w):
    """General invertible pull maps (random Def 4.14 memory layouts, R2, whose Q
    scatters the low bits; and a transpose into a Def 4.11 swizzle): planned as linear
    CTA tiles (XOR-addressed src vectors, coalesced runs on both sides, smem / shuffle
    exchange), never the generic kernel; bit-exact against the oracle."""
    import torch
    rng = np.random.default_rng(300 + w)
    cases = []
    for d in (14, 17, 20):
        cases.append(([("offset", d)], [("x", d)], gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)))
    m = n = 9
    S = ll.ll_layout_mma_swizzle(m, n, 1, 1, 8)             # Def 4.11, vec 1
    tcols = [(1 << (k + n)) if k < m else (1 << (k - m)) for k in range(m + n)]   # column-major
    cases.append(([("offset", m + n)], [tuple(x) for x in S.out_dims], tcols, S.cols()))
    for in_dims, out, ca, cb in cases:
        d = in_dims[0][1]
        OA, OB = O.layout_from_cols(in_dims, out, ca), O.layout_from_cols(in_dims, out, cb)
        A = ll.Layout(in_dims, out, {"offset": [O.logical_coords(out, c) for c in ca]})
        B = ll.Layout(in_dims, out, {"offset": [O.logical_coords(out, c) for c in cb]})
        plan = ll.ll_plan_convert(A, B, w)
        assert plan.describe()["exec"] == "tile", plan.describe()["exec"]
        src = gen.random_bits(rng, 1 << d, w)
        d_dst = empty_device(1 << d, w)
        ll.ll_convert(to_device(src), d_dst, plan)
        torch.cuda.synchronize()
        assert np.array_equal(from_device(d_dst, w), O.convert(OA, OB, src)), d


@pytest.mark.gpu
def test_e1_exhaustive_generic_gpu():
    """E1 on the GPU, exhaustive: all 8! = 40320 bijective relabelings B
    of Fig. 1's 2^8 space against Fig. 1 A, each executed by the runtime-generic
    kernel (XOR-of-columns pull map) into its own slice of one device buffer, then
    compared in one go with the oracle's pack_B(T)."""
    import itertools
    import torch
    A, OA = both(W.C1_A)
    T = gen.random_bits(np.random.default_rng(1001), 256, 4)
    d_src = to_device(O.pack(OA, T))
    unit = [1 << t for t in range(8)]
    perms = list(itertools.permutations(range(8)))
    d_dst = torch.empty((len(perms), 256), dtype=torch.int32, device="cuda")
    want = np.empty((len(perms), 256), dtype=np.uint32)
    for case, perm in enumerate(perms):
        OB = O.layout_from_cols(OA.in_dims, OA.out_dims, [unit[p] for p in perm])
        B = ll.Layout(OB.in_dims, OB.out_dims, OB.bases)
        plan = ll.ll_plan_convert(A, B, 4, generic=True)
        ll.ll_convert(d_src, d_dst[case], plan)
        want[case] = O.pack(OB, T)
    torch.cuda.synchronize()
    got = d_dst.cpu().numpy().view(np.uint32)
    bad = np.nonzero(~np.all(got == want, axis=1))[0]
    assert bad.size == 0, [perms[i] for i in bad[:5]]


@pytest.mark.parametrize("which", ["n2", "c1b", "c3", "acc_fp8"])
def test_autotune_bitexact(which):
    """ll_plan_autotune: every candidate decomposition (incl. faithful σ and the permuted
    sub-word shuffle) is timed on the caller's buffers; the returned (fastest) plan
    converts bit-exactly, and describe lists the candidates."""
    sa, sb, w = {"n2": (*W.n2_tmem_epilogue(5), 4), "c1b": (*W.c1_batched(8), 4), "c3": (*W.c3(3), 2),
                 "acc_fp8": (*W.n2_acc_to_lhs(8, 6), 1)}[which]
    A, OA = both(sa)
    B, OB = both(sb)
    T = gen.random_bits(np.random.default_rng(12), 1 << OA.d_out, w)
    src = O.pack(OA, T)
    d_src, d_dst = to_device(src), empty_device(1 << OB.d_in, w)
    plan = ll.ll_plan_autotune(A, B, w, d_src, d_dst, iters=3)
    cands = plan.describe()["autotune"]
    assert len(cands) >= 2 and all(c["ms"] > 0 for c in cands)
    d_dst.zero_()
    ll.ll_convert(d_src, d_dst, plan)
    assert np.array_equal(from_device(d_dst, w), O.pack(OB, T))


# ---------------------------------------------------------------- N3: scans
@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("sigma", ["coalesced", "faithful"])
def test_scan_bitexact(family, sigma):
    """O13: in-tile inclusive scan along the axis (§8(f) N3) on config-4 tiles —
    bit-equal to the oracle's fixed-order fp32 recurrence (defined in logical
    coordinates, so independent of σ) and within 7·2^-24 of the fp64 prefix sums."""
    import torch
    spec = W.c4("reduce", family, n_i=9, n_j=9)
    L, OL = both(spec)
    T = np.random.default_rng(1007).random(1 << OL.d_out, dtype=np.float32)
    src = O.pack(OL, T)
    plan = ll.ll_plan_scan(L, 1, sigma=sigma)
    out = torch.empty(src.size, dtype=torch.float32, device="cuda")
    ll.ll_scan(torch.from_numpy(src).cuda(), out, plan)
    got = out.cpu().numpy()
    rep = O.scan_bitdoubling_fp32(OL, 1, src)
    assert np.array_equal(got.view(np.uint32), rep.view(np.uint32))
    ref = O.scan_ref_fp64(OL, 1, src)
    assert np.all(np.abs(got - ref) <= 7 * 2.0 ** -24 * np.abs(ref) + 1e-30)


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("pipe", ["auto", "bulk"])
def test_scan_fullsize_tma_store(family, pipe):
    """Config-4 scan on the whole [4096, 4096] fp32 tensor in [128, 128] tiles, in the
    bench's launch configuration (auto: direct 16-byte loads and stores, 16 warps) and
    with TMA stages (bulk: tiles in by cp.async.bulk, results back through the stage and
    out by cp.async.bulk): every element bit-equal to the oracle's fixed-order recurrence."""
    import torch
    spec = W.c4("reduce", family)
    L, OL = both(spec)
    plan = ll.ll_plan_scan(L, 1, pipe=pipe)
    d = plan.describe()
    if pipe == "bulk":
        assert d["tma"] and d["tma_store"]        # 1024 tiles: the bulk-store path
    else:
        assert not d["tma"] and d["warp_bits"] == 4
    T = np.random.default_rng(1008).random(1 << OL.d_out, dtype=np.float32)
    src = O.pack(OL, T)
    out = torch.empty(src.size, dtype=torch.float32, device="cuda")
    ll.ll_scan(torch.from_numpy(src).cuda(), out, plan)
    rep = O.scan_bitdoubling_fp32(OL, 1, src)
    assert np.array_equal(out.cpu().numpy().view(np.uint32), rep.view(np.uint32))


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("op", ["max", "min"])
def test_scan_max_min_bitexact(family, op):
    """Running max / min (ll_plan_opts.reduce_op) along the axis inside [128,128] tiles,
    plus the warp-crossing (smem) steps of a layout with axis bits on the warps: exact,
    so bit-equal to the oracle's fp64 running max / min."""
    import torch
    rng = np.random.default_rng(1011)
    warp_axis = {"out": [("b", 3), ("i", 5), ("j", 7)],
                 "in": [("reg", ["j0", "j1", "j2"]), ("lane", ["i0", "i1", "i2", "i3", "i4"]),
                        ("warp", ["j3", "j4", "j5", "j6"]), ("block", ["b0", "b1", "b2"])]}
    for spec, axis in ((W.c4("reduce", family, n_i=9, n_j=9), 1), (warp_axis, 2)):
        L, OL = both(spec)
        T = (rng.random(1 << OL.d_out, dtype=np.float32) - 0.5).astype(np.float32)
        src = O.pack(OL, T)
        for sigma in ("coalesced", "faithful"):
            plan = ll.ll_plan_scan(L, axis, sigma=sigma, reduce_op=op)
            assert plan.describe()["op"] == op
            out = torch.empty(src.size, dtype=torch.float32, device="cuda")
            ll.ll_scan(torch.from_numpy(src).cuda(), out, plan)
            ref = O.scan_ref_fp64(OL, axis, src, op).astype(np.float32)
            assert np.array_equal(out.cpu().numpy().view(np.uint32), ref.view(np.uint32)), (sigma, axis)


@pytest.mark.parametrize("family", ["blocked", "mma", "mma_input", "sliced_blocked", "sliced_mma",
                                    "sliced_mma_input", "custom"])
def test_table4_scan_families(family):
    """§8(f) N3: scans along either dim over every Table 4 family and shape —
    steps over registers, lanes and (through shared memory) warps — including broadcast
    layouts whose duplicated positions must all hold the same value: bit-exact
    against the fixed-order replica, packed like the input."""
    import torch
    rng = np.random.default_rng(4848)
    ran = 0
    for shape in TABLE4_SHAPES:
        OL, L = _table4_layout(family, shape, rng)
        T = rng.random(1 << OL.d_out, dtype=np.float32)
        src = O.pack(OL, T)
        for axis in (1, 0):
            try:
                plan = ll.ll_plan_scan(L, axis)
            except ll.LLError as e:
                # the only refusal: a warp-crossing step whose exchange buffer (one value
                # per thread and register) exceeds shared memory (the 512-register custom tile)
                assert "too large" in str(e), (family, shape, axis, e)
                continue
            rep = O.scan_bitdoubling_fp32(OL, axis, src)
            # default plan (direct loads), then TMA stages with the bulk store (pipe = bulkst)
            for p in (plan, ll.ll_plan_scan(L, axis, pipe="bulkst")):
                out = torch.empty(src.size, dtype=torch.float32, device="cuda")
                ll.ll_scan(torch.from_numpy(src).cuda(), out, p)
                got = out.cpu().numpy()
                assert np.array_equal(got.view(np.uint32), rep.view(np.uint32)), (family, shape, axis)
            ran += 1
    assert ran >= 8


def test_scan_axis_over_warps():
    """Scan steps over warp bits (shared-memory exchange) and over lanes and registers in
    one tile: axis j = (reg j0..j2, warp j3..j6) on a 512-thread CTA."""
    import torch
    spec = {"out": [("b", 3), ("i", 5), ("j", 7)],
            "in": [("reg", ["j0", "j1", "j2"]), ("lane", ["i0", "i1", "i2", "i3", "i4"]),
                   ("warp", ["j3", "j4", "j5", "j6"]), ("block", ["b0", "b1", "b2"])]}
    L, OL = both(spec)
    T = np.random.default_rng(1010).random(1 << OL.d_out, dtype=np.float32)
    src = O.pack(OL, T)
    for sigma in ("coalesced", "faithful"):
        plan = ll.ll_plan_scan(L, 2, sigma=sigma)
        out = torch.empty(src.size, dtype=torch.float32, device="cuda")
        ll.ll_scan(torch.from_numpy(src).cuda(), out, plan)
        rep = O.scan_bitdoubling_fp32(OL, 2, src)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), rep.view(np.uint32)), sigma


def test_gather_axis_over_warps_smem():
    """Gather with in-tile axis bits on the warps (L_Wrp^axis != 0, outside the paper's
    shuffle gather): the shared-memory gather over the staged tile, bit-exact."""
    import torch
    spec = {"out": [("b", 3), ("i", 5), ("j", 7)],
            "in": [("reg", ["j0", "j1", "j2"]), ("lane", ["i0", "i1", "i2", "i3", "i4"]),
                   ("warp", ["j3", "j4", "j5", "j6"]), ("block", ["b0", "b1", "b2"])]}
    L, OL = both(spec)
    rng = np.random.default_rng(1011)
    n = 1 << OL.d_in
    src = O.pack(OL, gen.random_bits(rng, n, 4))
    idx = O.pack(OL, rng.integers(-500, 500, size=n).astype(np.int32))
    with pytest.raises(ll.LLError, match="warps"):
        ll.ll_plan_gather(L, 2, 4, force_class="SHUFFLE")
    plan = ll.ll_plan_gather(L, 2, 4)
    assert plan.describe()["exchange"] == "smem"
    d_dst = empty_device(n, 4)
    ll.ll_gather(to_device(src), to_device(idx.view(np.uint32)), d_dst, plan)
    assert np.array_equal(from_device(d_dst, 4), O.gather(OL, 2, src, idx))


@pytest.mark.gpu
@pytest.mark.parametrize("grid_per_sm", [None, "1"])
@pytest.mark.parametrize("pipe", ["0", "1"])
def test_smem_pipeline_both_ways_gpu(monkeypatch, pipe, grid_per_sm):
    """The software-pipelined smem exchange (next tile's loads before this tile's smem
    reads and stores; pipe = "on" / LL_PIPE=1) and the plain one
    are both bit-exact against the oracle: config 3, config 1-batch (smem forced) and
    random R2 memory layouts planned as linear tiles.  LL_GRID_PER_SM=1 caps the grid at
    one CTA per SM, so every CTA loops over several tiles (the pipelined path's
    steady state)."""
    import torch
    monkeypatch.setenv("LL_PIPE", pipe)
    if grid_per_sm:
        monkeypatch.setenv("LL_GRID_PER_SM", grid_per_sm)
    else:
        monkeypatch.delenv("LL_GRID_PER_SM", raising=False)
    for (sa, sb), w, opts in [(W.c3(9), 2, {}), (W.c1_batched(12), 4, {"force_class": "SMEM"})]:
        A, OA = both(sa)
        B, OB = both(sb)
        plan = ll.ll_plan_convert(A, B, w, **opts)
        assert plan.describe()["tile"]["pipe"] == (pipe == "1")
        src = O.pack(OA, gen.random_bits(np.random.default_rng(1003), 1 << OA.d_out, w))
        d_dst = empty_device(src.size, w)
        ll.ll_convert(to_device(src), d_dst, plan)
        torch.cuda.synchronize()
        assert np.array_equal(from_device(d_dst, w), O.convert(OA, OB, src))
    rng = np.random.default_rng(800)
    linear = 0
    for w in (2, 4):
        for d in (16, 20):
            ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
            ins, out = [("offset", d)], [("x", d)]
            OA, OB = O.layout_from_cols(ins, out, ca), O.layout_from_cols(ins, out, cb)
            A = ll.Layout(ins, out, {"offset": [(c,) for c in ca]})
            B = ll.Layout(ins, out, {"offset": [(c,) for c in cb]})
            plan = ll.ll_plan_convert(A, B, w)
            t = plan.describe()
            if t["exec"] != "tile" or t["tile"]["xchg"] != "smem":
                continue
            linear += 1
            assert t["tile"]["pipe"] == (pipe == "1")
            src = gen.random_bits(rng, 1 << d, w)
            d_dst = empty_device(1 << d, w)
            ll.ll_convert(to_device(src), d_dst, plan)
            torch.cuda.synchronize()
            assert np.array_equal(from_device(d_dst, w), O.convert(OA, OB, src)), (w, d)
    assert linear >= 2



@pytest.mark.parametrize("w", [2, 4])
def test_linear_tile_register_cap_and_autotune_gpu(w):
    """Linear tiles under every pipe x min_blocks variant (the ptxas register cap makes
    the kernel spill) and the plan ll_plan_autotune picks among them: bit-exact against
    the oracle on random R2 memory layouts."""
    import torch
    rng = np.random.default_rng(900 + w)
    d = 20
    ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
    ins, out = [("offset", d)], [("x", d)]
    OA, OB = O.layout_from_cols(ins, out, ca), O.layout_from_cols(ins, out, cb)
    A = ll.Layout(ins, out, {"offset": [(c,) for c in ca]})
    B = ll.Layout(ins, out, {"offset": [(c,) for c in cb]})
    src = gen.random_bits(rng, 1 << d, w)
    ref = O.convert(OA, OB, src)
    d_src = to_device(src)
    for pipe in ("off", "on"):
        for mb in (-1, 2, 3):
            plan = ll.ll_plan_convert(A, B, w, pipe=pipe, min_blocks=mb)
            assert plan.describe()["tile"]["linear_tile"]
            d_dst = empty_device(1 << d, w)
            ll.ll_convert(d_src, d_dst, plan)
            torch.cuda.synchronize()
            assert np.array_equal(from_device(d_dst, w), ref), (pipe, mb)
    d_dst = empty_device(1 << d, w)
    plan = ll.ll_plan_autotune(A, B, w, d_src, d_dst, iters=2)
    tune = plan.describe().get("autotune", [])
    assert any(c.get("min_blocks") == 2 for c in tune) and any(c.get("pipe") is False for c in tune)
    d_dst.zero_()
    ll.ll_convert(d_src, d_dst, plan)
    torch.cuda.synchronize()
    assert np.array_equal(from_device(d_dst, w), ref)


def test_staged_exchange_gpu():
    """The staged smem exchange (ll_plan_opts.pipe = "staged": the next two tiles' src
    vectors streamed by cp.async into two raw smem stages, persistent grid, so every CTA
    loops over several tiles) is bit-exact against the oracle on config 3, config
    1-batch (smem forced) and random R2 memory layouts (linear tiles), and autotune
    times it for linear tiles."""
    import torch
    for (sa, sb), w, opts in [(W.c3(9), 2, {}), (W.c1_batched(14), 4, {"force_class": "SMEM"})]:
        A, OA = both(sa)
        B, OB = both(sb)
        plan = ll.ll_plan_convert(A, B, w, pipe="staged", **opts)
        assert plan.describe()["tile"]["staged"] is True
        src = O.pack(OA, gen.random_bits(np.random.default_rng(1007), 1 << OA.d_out, w))
        d_dst = empty_device(src.size, w)
        ll.ll_convert(to_device(src), d_dst, plan)
        torch.cuda.synchronize()
        assert np.array_equal(from_device(d_dst, w), O.convert(OA, OB, src))
    rng = np.random.default_rng(810)
    for w in (1, 2, 4, 8):
        for d in (18, 22):
            ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
            ins, out = [("offset", d)], [("x", d)]
            OA, OB = O.layout_from_cols(ins, out, ca), O.layout_from_cols(ins, out, cb)
            A = ll.Layout(ins, out, {"offset": [(c,) for c in ca]})
            B = ll.Layout(ins, out, {"offset": [(c,) for c in cb]})
            plan = ll.ll_plan_convert(A, B, w, pipe="staged")
            t = plan.describe()
            if t["exec"] != "tile" or t["tile"]["xchg"] != "smem":
                continue
            src = gen.random_bits(rng, 1 << d, w)
            d_src = to_device(src)
            d_dst = empty_device(1 << d, w)
            ll.ll_convert(d_src, d_dst, plan)
            torch.cuda.synchronize()
            ref = O.convert(OA, OB, src)
            assert np.array_equal(from_device(d_dst, w), ref), (w, d, t["tile"]["staged"])
            if w == 4 and d == 22:
                tuned = ll.ll_plan_autotune(A, B, w, d_src, d_dst, iters=2)
                assert any(c.get("staged") for c in tuned.describe().get("autotune", []))
                d_dst.zero_()
                ll.ll_convert(d_src, d_dst, tuned)
                torch.cuda.synchronize()
                assert np.array_equal(from_device(d_dst, w), ref)


@pytest.mark.parametrize("cfg", ["c3", "c3b"])
@pytest.mark.parametrize("pipe", ["bulk", "bulkst"])
def test_bulk_staged_smem_exchange_full_size(cfg, pipe):
    """The bulk-staged smem exchange (src tiles by cp.async.bulk into raw stages; with
    bulkst the dst tiles also leave by cp.async.bulk) on configs 3 / 3b at full size:
    every element against H(B(h)) and sampled outputs against the oracle."""
    sa, sb = {"c3": W.c3(14), "c3b": W.c3b(14)}[cfg]
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    d = ll.ll_plan_convert(A, B, 2, pipe=pipe).describe()
    assert d["tile"]["bulk"] == ("load" if pipe == "bulk" else "load+store")
    _full_size_every_element_opts(sa, sb, 2, 1013, pipe=pipe)


def test_permuted_subword_shuffles_gpu():
    """The element-permuted sub-word shuffles (reading R-V) on random SHUFFLE-class pairs
    with 1- and 2-byte elements, batched over 8 tiles: bit-exact against the oracle."""
    rng = np.random.default_rng(31)
    out = [("i", 5), ("j", 5)]
    done = 0
    for case in range(400):
        r = int(rng.integers(3, 6))
        hw = [("reg", r), ("lane", 5), ("warp", 10 - r - 5)]
        sa = gen.random_distributed(rng, out, hw)
        sb = gen.random_distributed(rng, out, hw)
        for w in (1, 2):
            d = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w).describe()
            if not d.get("tile", {}).get("element_permutes"):
                continue
            ba = {"out": [("b", 3)] + list(sa["out"]), "in": list(sa["in"]) + [("block", ["b0", "b1", "b2"])]}
            bb = {"out": [("b", 3)] + list(sb["out"]), "in": list(sb["in"]) + [("block", ["b0", "b1", "b2"])]}
            got, ref, plan = run_convert(ba, bb, w, case)
            assert plan.describe()["tile"]["element_permutes"]
            assert np.array_equal(got, ref), (case, w)
            done += 1
        if done >= 24:
            break
    assert done >= 5


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("thread_bytes", [256, 128])
def test_reduce_scan_more_warps_bitexact(family, thread_bytes):
    """Non-axis register bits moved to extra warps (ll_plan_opts.thread_bytes: 8 / 16
    warps per [128,128] tile): reduce bit-exact against the logical-order replica and
    scan against the bit-doubling recurrence — the orders do not depend on the kernel
    layout."""
    import torch
    L, OL = both(W.c4("reduce", family, n_i=9, n_j=9))
    T = np.random.default_rng(1009).random(1 << OL.d_out, dtype=np.float32)
    src = O.pack(OL, T)
    d_src = torch.from_numpy(src).cuda()
    p = ll.ll_plan_reduce(L, 1, thread_bytes=thread_bytes)
    assert p.describe()["warp_bits"] > 2
    out = torch.empty(p.out_elems(), dtype=torch.float32, device="cuda")
    ll.ll_reduce(d_src, out, p)
    rep = O.reduce_fixed_order_fp32(OL, 1, src)
    assert np.array_equal(out.cpu().numpy().view(np.uint32), rep.view(np.uint32))
    s = ll.ll_plan_scan(L, 1, thread_bytes=thread_bytes)
    assert s.describe()["warp_bits"] > 2
    out2 = torch.empty(src.size, dtype=torch.float32, device="cuda")
    ll.ll_scan(d_src, out2, s)
    rep2 = O.scan_bitdoubling_fp32(OL, 1, src)
    assert np.array_equal(out2.cpu().numpy().view(np.uint32), rep2.view(np.uint32))


@pytest.mark.parametrize("family", ["mma", "blocked"])
@pytest.mark.parametrize("thread_bytes", [64, 32])
def test_gather_more_warps_bitexact(family, thread_bytes):
    """Gather with non-axis register bits moved to extra warps (thread_bytes): O10."""
    from tests._util import from_device, to_device, empty_device
    rng = np.random.default_rng(1010)
    L, OL = both(W.c4("gather", family, n_i=9, n_j=7))
    n = 1 << OL.d_in
    src = O.pack(OL, gen.random_bits(rng, n, 4))
    idx = O.pack(OL, rng.integers(-50, 50, size=n).astype(np.int32))
    plan = ll.ll_plan_gather(L, 1, 4, thread_bytes=thread_bytes)
    assert plan.describe()["warp_bits"] >= 2
    d_dst = empty_device(n, 4)
    ll.ll_gather(to_device(src), to_device(idx.view(np.uint32)), d_dst, plan)
    assert np.array_equal(from_device(d_dst, 4), O.gather(OL, 1, src, idx))


@pytest.mark.parametrize("family", ["mma", "blocked", "sliced_mma", "custom"])
@pytest.mark.parametrize("tile_bytes", [16384, 4096])
def test_split_tiles_bitexact(family, tile_bytes):
    """Smaller CTA tiles (ll_plan_opts.tile_bytes): warp bits carrying independent rows
    become grid bits.  Reduce, scan (both axes, [128,128] Table 4 tiles x 4 CTAs) and
    gather (config-4 tiles) stay bit-exact against the oracle: the reduction / scan /
    gather never crosses those bits."""
    import torch
    from tests._util import from_device, to_device, empty_device
    rng = np.random.default_rng(1012)
    OT, _ = _table4_layout(family, (128, 128), rng)
    # 4 CTAs along a new leading dim (block bits)
    out3 = [("b", 2)] + list(OT.out_dims)
    bases = {n: [(0,) + tuple(v) for v in OT.bases[n]] for n, _ in OT.in_dims}
    bases["block"] = [(1, 0, 0), (2, 0, 0)]
    OL = O.Layout(list(OT.in_dims) + [("block", 2)], out3, bases)
    L = ll.Layout(OL.in_dims, OL.out_dims, OL.bases)
    T = rng.random(1 << OL.d_out, dtype=np.float32)
    src = O.pack(OL, T)
    d_src = torch.from_numpy(src).cuda()
    split = 0
    for axis in (1, 2):
        p0 = ll.ll_plan_reduce(L, axis)
        p = ll.ll_plan_reduce(L, axis, tile_bytes=tile_bytes)
        split += p.describe()["ctas"] > p0.describe()["ctas"]
        out = torch.empty(p.out_elems(), dtype=torch.float32, device="cuda")
        ll.ll_reduce(d_src, out, p)
        rep = O.reduce_fixed_order_fp32(OL, axis, src)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), rep.view(np.uint32)), (family, axis)
        try:
            s = ll.ll_plan_scan(L, axis, tile_bytes=tile_bytes)
        except ll.LLError as e:
            assert "too large" in str(e)
            continue
        out2 = torch.empty(src.size, dtype=torch.float32, device="cuda")
        ll.ll_scan(d_src, out2, s)
        rep2 = O.scan_bitdoubling_fp32(OL, axis, src)
        assert np.array_equal(out2.cpu().numpy().view(np.uint32), rep2.view(np.uint32)), (family, axis)
    assert split >= 1
    if family in ("mma", "blocked"):
        G, OG = both(W.c4("gather", family, n_i=9, n_j=7))
        n = 1 << OG.d_in
        gs = O.pack(OG, gen.random_bits(rng, n, 4))
        gi = O.pack(OG, rng.integers(-50, 50, size=n).astype(np.int32))
        for fc in (None, "SMEM"):
            g = ll.ll_plan_gather(G, 1, 4, tile_bytes=tile_bytes, force_class=fc)
            d_dst = empty_device(n, 4)
            ll.ll_gather(to_device(gs), to_device(gi.view(np.uint32)), d_dst, g)
            assert np.array_equal(from_device(d_dst, 4), O.gather(OG, 1, gs, gi)), (family, fc)
