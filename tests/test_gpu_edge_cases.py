"""Edge cases of the GPU path against the oracle (-m gpu).

* Degenerate sizes: 0- to 6-bit layouts (one element up to less than a warp's worth;
  tile kernels need >= 32 elements, below that the generic kernel runs), and a single
  warp with no register or warp bits.
* Maximum sizes: buffers beyond 2^32 bytes / 2^31 elements, so every byte offset
  needs 64 bits — conversion (config-2 layouts, 2^18 tiles: 8 GiB in + 8 GiB out),
  gather (2^31 fp32 elements) and reduce (2^31 fp32 elements), checked on sampled
  outputs one by one (conversion, gather) or per-output against fp64 (reduce).
* No ragged inputs exist: linear layouts describe power-of-two shapes only (P:128,
  limitation stated at P:565); every dimension size is 2^k, so "tails" are whole tiles.
"""
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


@pytest.mark.parametrize("d", range(0, 7))
@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_tiny_memory_layouts(d, w):
    rng = np.random.default_rng(100 * d + w)
    out = [("x", d)]
    cols_b = gen.random_memory_cols(rng, d) if d else []
    OA = O.Layout([("offset", d)], out, {"offset": [[1 << k] for k in range(d)]})
    OB = O.layout_from_cols([("offset", d)], out, cols_b)
    A = ll.Layout(OA.in_dims, OA.out_dims, OA.bases)
    B = ll.Layout(OB.in_dims, OB.out_dims, OB.bases)
    T = gen.random_bits(rng, 1 << d, w)
    src = O.pack(OA, T)
    for A_, B_, OA_, OB_, s in ((A, B, OA, OB, src), (B, A, OB, OA, O.pack(OB, T))):
        plan = ll.ll_plan_convert(A_, B_, w)
        d_dst = empty_device(1 << d, w)
        ll.ll_convert(to_device(s), d_dst, plan)
        assert np.array_equal(from_device(d_dst, w), O.convert(OA_, OB_, s)), plan.describe()["exec"]


def test_single_warp_no_registers():
    """reg = 0 bits, one warp, lanes permuted (x0..x4 reversed): a pure shuffle."""
    spec_a = {"out": [("x", 5)], "in": [("reg", []), ("lane", ["x0", "x1", "x2", "x3", "x4"]), ("warp", [])]}
    spec_b = {"out": [("x", 5)], "in": [("reg", []), ("lane", ["x4", "x3", "x2", "x1", "x0"]), ("warp", [])]}
    A, OA = both(spec_a)
    B, OB = both(spec_b)
    for w in (1, 2, 4, 8):
        T = gen.random_bits(np.random.default_rng(w), 32, w)
        src = O.pack(OA, T)
        plan = ll.ll_plan_convert(A, B, w)
        d_dst = empty_device(32, w)
        ll.ll_convert(to_device(src), d_dst, plan)
        assert np.array_equal(from_device(d_dst, w), O.pack(OB, T))


def _sample(n, rng, k=1 << 18):
    """Sampled indices: random, both ends, and around every 2^31 / 2^32 boundary."""
    edges = [0, n - 4096]
    for b in (31, 32, 33):
        if (1 << b) < n:
            edges += [(1 << b) - 2048]
    hs = [rng.integers(0, n, size=k)] + [e + np.arange(4096) for e in edges]
    return np.unique(np.concatenate(hs)).astype(np.uint64)


def test_max_size_convert_8gib():
    """Config-2 layouts with 2^18 tiles: 2^32 bf16 elements = 8 GiB in + 8 GiB out."""
    import torch
    sa, sb = W.c2(18)
    A, OA = both(sa)
    B, OB = both(sb)
    plan = ll.ll_plan_convert(A, B, 2)
    from workloads import hashfill as H
    n = 1 << 32
    src = H.fill(sa, 2, 1002)
    dst = torch.empty_like(src)
    ll.ll_convert(src, dst, plan)
    torch.cuda.synchronize()
    assert H.check(sb, 2, 1002, dst) == 0          # every one of the 2^32 elements
    hs = _sample(n, np.random.default_rng(5))
    hsrc = O.apply_inverse_all(OA, O.apply_all(OB, hs)).astype(np.int64)
    got = dst[torch.from_numpy(hs.astype(np.int64)).cuda()].cpu().numpy()
    want = src[torch.from_numpy(hsrc).cuda()].cpu().numpy()
    assert np.array_equal(got, want)
    del src, dst
    torch.cuda.empty_cache()


def test_max_size_gather_8gib():
    """Config-4 gather tiles [128, 32] (MMA) over a [2^16, 2^15] fp32 tensor: 2^31
    elements, 8 GiB each of src, idx and dst; sampled outputs against O10 applied
    point by point (out[x] = src[x with the axis coordinate's low K bits := idx[x]])."""
    import torch
    spec = W.c4("gather", "mma", n_i=16, n_j=15, k_bits=5)
    L, OL = both(spec)
    n = 1 << OL.d_in
    plan = ll.ll_plan_gather(L, 1, 4)
    g = torch.Generator(device="cuda").manual_seed(1004)
    src = torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda", generator=g)
    idx = torch.randint(-1000, 1000, (n,), dtype=torch.int32, device="cuda", generator=g)
    dst = torch.empty_like(src)
    ll.ll_gather(src, idx, dst, plan)
    torch.cuda.synchronize()
    hs = _sample(n, np.random.default_rng(6))
    th = torch.from_numpy(hs.astype(np.int64)).cuda()
    x = O.apply_all(OL, hs)                        # logical flat index of each output
    nj = 15
    j = x & np.uint64((1 << nj) - 1)
    K = np.uint64(32)
    k = idx[th].cpu().numpy().astype(np.int64) & 31   # G16: masked to [0, K)
    xs = (x - j) | ((j & ~(K - np.uint64(1))) | k.astype(np.uint64))
    hsrc = O.apply_inverse_all(OL, xs).astype(np.int64)
    got = dst[th].cpu().numpy()
    want = src[torch.from_numpy(hsrc).cuda()].cpu().numpy()
    assert np.array_equal(got, want)
    del src, idx, dst
    torch.cuda.empty_cache()


def test_max_size_reduce_8gib():
    """Config-4 reduce tiles [128, 128] (blocked) over a [2^16, 2^15] fp32 tensor:
    2^31 inputs (8 GiB) -> [2^16, 2^8]; sampled outputs within 1e-6 of the fp64 sum of
    their 128 inputs, located through the oracle's inverse (O11)."""
    import torch
    spec = W.c4("reduce", "blocked", n_i=16, n_j=15)
    L, OL = both(spec)
    n = 1 << OL.d_in
    plan = ll.ll_plan_reduce(L, 1)
    g = torch.Generator(device="cuda").manual_seed(1005)
    src = torch.rand((n,), dtype=torch.float32, device="cuda", generator=g)
    out = torch.empty(plan.out_elems(), dtype=torch.float32, device="cuda")
    assert plan.out_elems() == (1 << 16) * (1 << 8)
    ll.ll_reduce(src, out, plan)
    torch.cuda.synchronize()
    rng = np.random.default_rng(7)
    ys = np.unique(np.concatenate([rng.integers(0, out.numel(), size=4096), np.arange(64),
                                   out.numel() - 1 - np.arange(64)])).astype(np.uint64)
    # output y = (i, jt) row-major over [2^16, 2^8]; its inputs are j = jt*128 + t
    i, jt = ys >> np.uint64(8), ys & np.uint64(255)
    t = np.arange(128, dtype=np.uint64)
    xs = ((i[:, None] << np.uint64(15)) | (jt[:, None] << np.uint64(7)) | t[None, :]).reshape(-1)
    hs = O.apply_inverse_all(OL, xs).astype(np.int64)
    vals = src[torch.from_numpy(hs).cuda()].cpu().numpy().astype(np.float64).reshape(-1, 128)
    ref = vals.sum(axis=1)
    got = out[torch.from_numpy(ys.astype(np.int64)).cuda()].cpu().numpy()
    assert np.all(np.abs(got - ref) <= 1e-6 * np.abs(ref))
    del src, out
    torch.cuda.empty_cache()


@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_random_memory_layouts_gpu(w):
    """R2 random memory layouts (Def 4.14) <-> row-major on the GPU, d = 8..14: the
    XOR-copy tiles (and the generic kernel where the low bits scatter) bit-exact."""
    for d in (8, 10, 12, 14):
        for seed in range(4):
            rng = np.random.default_rng(seed * 31 + d + 100 * w)
            out = [("x", d)]
            OA = O.Layout([("offset", d)], out, {"offset": [[1 << k] for k in range(d)]})
            OB = O.layout_from_cols([("offset", d)], out, gen.random_memory_cols(rng, d))
            A = ll.Layout(OA.in_dims, OA.out_dims, OA.bases)
            B = ll.Layout(OB.in_dims, OB.out_dims, OB.bases)
            T = gen.random_bits(rng, 1 << d, w)
            for A_, B_, OA_, OB_ in ((A, B, OA, OB), (B, A, OB, OA)):
                s = O.pack(OA_, T)
                plan = ll.ll_plan_convert(A_, B_, w)
                d_dst = empty_device(1 << d, w)
                ll.ll_convert(to_device(s), d_dst, plan)
                assert np.array_equal(from_device(d_dst, w), O.convert(OA_, OB_, s)), (d, seed, plan.describe()["exec"])
