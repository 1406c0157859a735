"""Broadcast conversions on the GPU (P:306-308 zero columns; rule (2) P:358-362):
random bijective A -> B with 1-8 zero columns (replica bits on registers, lanes and
warps), batched.  Every dst element (every replica) equals the closed form H(B(h)) of
hash-filled src (O5), and the executed kernel is the specialised tile kernel.  Small
cases are also compared with the oracle's conversion directly."""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen
from workloads import hashfill as H

pytestmark = pytest.mark.gpu

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


@pytest.mark.parametrize("n_zero", [1, 2, 4, 5, 6, 7, 8])
@pytest.mark.parametrize("w", [1, 2, 4, 8])
def test_broadcast_replicas_bitexact(n_zero, w):
    import torch
    from tests._util import to_device
    rng = np.random.default_rng(7000 + 10 * n_zero + w)
    for case in range(3):
        sa, sb = gen.random_broadcast_pair(rng, n_zero, batch_bits=3)
        A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
        OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
        p = ll.ll_plan_convert(A, B, w)
        assert p.describe()["exec"] == "tile"
        T = gen.random_bits(rng, 1 << OA.d_out, w)
        src = O.pack(OA, T)
        d_dst = torch.zeros((1 << OB.d_in) * w // 2 if w >= 2 else 1 << OB.d_in,
                            dtype=torch.int16 if w >= 2 else torch.uint8, device="cuda")
        ll.ll_convert(to_device(src), d_dst, p)
        got = d_dst.cpu().numpy().view(src.dtype)
        assert np.array_equal(got, O.convert(OA, OB, src)), (n_zero, w, case)


@pytest.mark.parametrize("n_zero", [5, 8])
def test_broadcast_large_every_element(n_zero):
    """~1 GiB of dst: every replica of every element against H(B(h))."""
    import torch
    rng = np.random.default_rng(8000 + n_zero)
    sa, sb = gen.random_broadcast_pair(rng, n_zero, ki=5, kj=5, batch_bits=18 - n_zero)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    p = ll.ll_plan_convert(A, B, 4)
    assert p.describe()["exec"] == "tile"
    src = H.fill(sa, 4, 5)
    dst = torch.zeros(1 << B.d_in, dtype=torch.int32, device="cuda")
    ll.ll_convert(src, dst, p)
    torch.cuda.synchronize()
    assert H.check(sb, 4, 5, dst) == 0


@pytest.mark.parametrize("n_zero", [2, 5, 8])
def test_broadcast_cta_class_bitexact(n_zero):
    """Broadcast targets with permuted block bits (CTA class), batched: bit-exact against
    the oracle, and at ~1 GiB every element against H(B(h))."""
    import torch
    from tests._util import to_device
    rng = np.random.default_rng(7100 + n_zero)
    for case in range(3):
        sa, sb = gen.random_broadcast_pair(rng, n_zero, batch_bits=4, permute_batch=True)
        OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
        p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 4)
        assert p.describe()["exec"] == "tile"
        src = O.pack(OA, gen.random_bits(rng, 1 << OA.d_out, 4))
        d_dst = torch.zeros(1 << OB.d_in, dtype=torch.int32, device="cuda")
        ll.ll_convert(to_device(src), d_dst, p)
        assert np.array_equal(d_dst.cpu().numpy().view(np.uint32), O.convert(OA, OB, src)), case
    sa, sb = gen.random_broadcast_pair(rng, n_zero, ki=5, kj=5, batch_bits=18 - n_zero, permute_batch=True)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    p = ll.ll_plan_convert(A, B, 4)
    src = H.fill(sa, 4, 9)
    dst = torch.zeros(1 << B.d_in, dtype=torch.int32, device="cuda")
    ll.ll_convert(src, dst, p)
    torch.cuda.synchronize()
    assert H.check(sb, 4, 9, dst) == 0
