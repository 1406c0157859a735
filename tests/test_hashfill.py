"""Pins for workloads/hashfill.py (the at-scale input generator and its closed-form
check) against the oracle's O2 apply / pack and a scalar splitmix64.
CPU only."""
import numpy as np
import pytest
import torch

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import hashfill as H


def test_splitmix64_tensor_matches_scalar():
    """Two's-complement torch arithmetic reproduces the unsigned 64-bit finaliser
    (published test value: splitmix64 stream from seed 0 starts 0xE220A8397B1DCDAF)."""
    assert H.splitmix64_scalar(0) == 0xE220A8397B1DCDAF
    xs = [0, 1, 2, 12345, (1 << 40) + 7, (1 << 63) - 1]
    got = H.splitmix64(torch.tensor(xs, dtype=torch.int64)).tolist()
    assert [g & ((1 << 64) - 1) for g in got] == [H.splitmix64_scalar(x) for x in xs]


SPECS = {
    "c1_A": W.C1_A,
    "c1_B": W.C1_B,
    "c2_A": W.c2(1)[0],
    "c2_B": W.c2(1)[1],
    "c4_mma": W.c4("reduce", "mma", n_i=8, n_j=8),
    "c5_A_p2": W.c5(2, n=6)[0],
    "c5_B_p2": W.c5(2, n=6)[1],
}


@pytest.mark.parametrize("name", sorted(SPECS))
@pytest.mark.parametrize("w", [2, 4])
def test_fill_is_pack_of_hash(name, w):
    """fill(spec) == O.pack(L, T) with T[x] = low w bytes of splitmix64(x ^ seed): the
    oracle's own packing of the hashed logical tensor."""
    spec = SPECS[name]
    L = O.Layout(*W.spec_to_bases(spec))
    seed = 77
    T = np.array([H.splitmix64_scalar(x ^ seed) & ((1 << (8 * w)) - 1) for x in range(1 << L.d_out)],
                 dtype=np.uint64).astype({2: np.uint16, 4: np.uint32}[w])
    want = O.pack(L, T)
    got = H.fill(spec, w, seed, device="cpu").numpy().view(want.dtype)
    assert np.array_equal(got, want)
    assert H.check(spec, w, seed, torch.from_numpy(want.view({2: np.int16, 4: np.int32}[w]).copy())) == 0


def test_fill_broadcast_layout_consistent():
    """A layout with zero columns gets equal bytes at every copy of a logical element
    (the A-consistency precondition of §8(b))."""
    spec = {"out": [("i", 2), ("j", 3)],
            "in": [("reg", ["j0", None]), ("lane", ["j1", "j2", "i0", "i1", None]), ("warp", [None])]}
    L = O.Layout(*W.spec_to_bases(spec))
    buf = H.fill(spec, 4, 5, device="cpu").numpy().view(np.uint32)
    assert O.is_consistent(L, buf)


def test_check_counts_mismatches():
    spec = W.C1_A
    buf = H.fill(spec, 4, 1, device="cpu")
    buf[3] ^= 1
    buf[200] ^= 1 << 20
    assert H.check(spec, 4, 1, buf) == 2
