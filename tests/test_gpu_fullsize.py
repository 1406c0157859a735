"""Every BASELINE config at its full size, in the launch configuration bench.py times
(the default plan, the same buffers' shapes), against the oracle (-m gpu).

Configs 2 and 3 are in test_gpu_convert.py.  Here: config 1 batch (2^20 tiles,
1 GiB), config 3b, config 4 gather and reduce for both families on the whole
[4096, 4096] fp32 tensor (every output compared with the oracle), config 5-T (2 GiB
transpose) and config 5 at P = 8 on the loopback communicator with both exchanges
(2 GiB).  Every element of every large conversion is compared on the device with the
closed form H(B(h)) of hash-filled src (O5 at scale, workloads/hashfill.py); 2^18-2^20
sampled outputs are additionally checked against the oracle's pull map point by point.
"""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen

pytestmark = pytest.mark.gpu

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def both(spec):
    return ll.Layout.from_spec(spec), O.Layout(*W.spec_to_bases(spec))


def _sampled(OA, OB, src, dst, n, seed, k=1 << 19):
    import torch
    rng = np.random.default_rng(seed)
    hs = np.unique(np.concatenate([rng.integers(0, n, size=k), np.arange(4096), n - 1 - np.arange(4096)]))
    hs = hs.astype(np.uint64)
    hsrc = O.apply_inverse_all(OA, O.apply_all(OB, hs)).astype(np.int64)
    got = dst[torch.from_numpy(hs.astype(np.int64)).cuda()].cpu().numpy()
    want = src[torch.from_numpy(hsrc).cuda()].cpu().numpy()
    assert np.array_equal(got, want)


@pytest.mark.parametrize("name", ["c1_batch", "c3b", "c5T"])
def test_fullsize_conversions(name):
    import torch
    (sa, sb), w = {"c1_batch": (W.c1_batched(20), 4), "c3b": (W.c3b(14), 2), "c5T": (W.c5T(0), 2)}[name]
    A, OA = both(sa)
    B, OB = both(sb)
    plan = ll.ll_plan_convert(A, B, w)
    from workloads import hashfill as H
    n = 1 << OA.d_in
    src = H.fill(sa, w, 1003)
    dst = torch.empty_like(src)
    ll.ll_convert(src, dst, plan)
    torch.cuda.synchronize()
    assert H.check(sb, w, 1003, dst) == 0
    _sampled(OA, OB, src, dst, n, 11)
    del src, dst
    torch.cuda.empty_cache()


@pytest.mark.parametrize("exchange", ["collective", "peer"])
def test_fullsize_config5_p8_loopback(exchange):
    """Config 5: [32768, 32768] bf16 row-sharded -> column-sharded over 8 virtual ranks
    (2 GiB); every element of every rank's slice against the closed form of O12."""
    import torch
    p, n = 3, 15
    sa, sb = W.c5(p, n=n)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    P = 1 << p
    plan = ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(P), exchange=exchange)
    total = 1 << (2 * n)
    nloc = total // P
    # src hash-filled: rank r's slice holds H(A(h, dev = r)); the closed form of O12 is
    # dst_r[h] = H(B(h, dev = r)), checked at every element of every rank's slice
    from workloads import hashfill as H
    seed = 1006
    src = H.fill(sa, 2, seed)
    dst = torch.empty_like(src)
    ws = torch.empty(max(16, plan.workspace_bytes()), dtype=torch.uint8, device="cuda")
    ll.ll_convert(src, dst, plan, workspace=ws)
    torch.cuda.synchronize()
    assert H.check(sb, 2, seed, dst) == 0
    # and sampled outputs of every rank against the oracle's O12 slice pull map
    rng = np.random.default_rng(13)
    for r in range(P):
        hs = np.concatenate([rng.integers(0, nloc, size=1 << 16), np.arange(1024), nloc - 1 - np.arange(1024)])
        hs = hs.astype(np.uint64)
        lb, offb = O.rank_slice(OB, r)
        xs = (O.apply_all(lb, hs) ^ np.uint64(offb))
        # the loopback src holds all ranks' slices back to back: A^+(x) is the global index
        hsrc = O.apply_inverse_all(OA, xs).astype(np.int64)
        got = dst[r * nloc + torch.from_numpy(hs.astype(np.int64)).cuda()]
        want = src[torch.from_numpy(hsrc).cuda()]
        assert torch.equal(got, want), r
    del src, dst
    torch.cuda.empty_cache()


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_fullsize_config4_gather(family):
    """Config 4 gather on the whole [4096, 4096] fp32 tensor in [128, 32] tiles: every
    output equal to O10 (take_along_axis inside each tile, indices masked, G16)."""
    import torch
    spec = W.c4("gather", family)
    L, OL = both(spec)
    n = 1 << OL.d_in
    rng = np.random.default_rng(1004)
    T = gen.random_bits(rng, n, 4)
    Ti = rng.integers(-1000, 1000, size=n).astype(np.int32)
    src, idx = O.pack(OL, T), O.pack(OL, Ti)
    plan = ll.ll_plan_gather(L, 1, 4)
    d_dst = torch.empty(n, dtype=torch.int32, device="cuda")
    ll.ll_gather(torch.from_numpy(src.view(np.int32)).cuda(), torch.from_numpy(idx).cuda(), d_dst, plan)
    got = d_dst.cpu().numpy().view(np.uint32)
    assert np.array_equal(got, O.gather(OL, 1, src, idx))


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_fullsize_config4_reduce(family):
    """Config 4 reduce on the whole [4096, 4096] fp32 tensor in [128, 128] tiles -> [4096,
    32]: every output within 1e-6 of the fp64 sum, and bit-equal to the fixed-order fp32
    replica on L (O11, reading R-reduce), for both kernel layouts σ."""
    import torch
    spec = W.c4("reduce", family)
    L, OL = both(spec)
    n = 1 << OL.d_in
    T = np.random.default_rng(1005).random(n, dtype=np.float32)
    src = O.pack(OL, T)
    plan = ll.ll_plan_reduce(L, 1)
    out = torch.empty(plan.out_elems(), dtype=torch.float32, device="cuda")
    ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan)
    got = out.cpu().numpy()
    ref = O.reduce_ref_fp64(OL, 1, src)
    assert got.size == 4096 * 32
    assert np.all(np.abs(got - ref) <= 1e-6 * np.abs(ref))
    rep = O.reduce_fixed_order_fp32(OL, 1, src)
    assert np.array_equal(got.view(np.uint32), rep.view(np.uint32))
    plan_f = ll.ll_plan_reduce(L, 1, sigma="faithful")
    out.fill_(-1.0)
    ll.ll_reduce(torch.from_numpy(src).cuda(), out, plan_f)
    assert np.array_equal(out.cpu().numpy().view(np.uint32), rep.view(np.uint32))
