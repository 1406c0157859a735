"""The C++17/OpenMP oracle (oracle/ll_oracle.cpp) against the numpy oracle and the
paper's fixed values, element by element (C++ file plus Python mirror).
CPU only."""
import numpy as np
import pytest

from oracle import cpp as OC
from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen


def L_of(spec):
    return O.Layout(*W.spec_to_bases(spec))


def test_builds_with_openmp():
    OC.build()
    assert OC.max_threads() >= 1


def test_table1_values():
    """GV1 (Table 1) through the C++ apply: (reg, thread) -> (i, j) under Fig. 1 A."""
    L = L_of(W.C1_A)
    pairs = {(0, 0): (0, 0), (1, 0): (0, 1), (0, 1): (0, 2), (1, 1): (0, 3), (2, 0): (1, 0),
             (3, 0): (1, 1), (0, 9): (2, 2), (1, 9): (2, 3), (2, 9): (3, 2), (3, 9): (3, 3)}
    hs = np.array([r | (t << 2) for (r, t) in pairs], dtype=np.uint64)
    xs = OC.apply(L.cols, hs)
    assert [(int(x) >> 4, int(x) & 15) for x in xs] == list(pairs.values())


@pytest.mark.parametrize("seed", range(6))
def test_right_inverse_and_min_preimage(seed):
    """O4: slack-zero right inverse == numpy's, and its images are the brute-force
    min-index preimages on random surjective matrices (R3)."""
    rng = np.random.default_rng(seed)
    d_out = int(rng.integers(3, 8))
    d_in = d_out + int(rng.integers(0, 4))
    while True:
        cols = [int(c) for c in rng.integers(0, 1 << d_out, size=d_in)]
        if O.rank(cols) == d_out:
            break
    L = O.layout_from_cols([("x", d_in)], [("y", d_out)], cols)
    inv = OC.right_inverse(cols, d_out)
    assert inv == O.right_inverse_cols(L)
    first = OC.preimage_min(cols, d_out)
    assert np.array_equal(first, O.preimage_min(L))
    for t in range(d_out):
        assert first[1 << t] == inv[t]


@pytest.mark.parametrize("cfg", ["c1", "c2", "c3", "c3b", "c5T"])
def test_convert_matches_numpy_oracle(cfg):
    """O5 on the configs at small batch: C++ (all threads and 1 thread) == numpy."""
    sa, sb = {"c1": (W.C1_A, W.C1_B), "c2": W.c2(2), "c3": W.c3(1), "c3b": W.c3b(1), "c5T": W.c5T(0, n=7)}[cfg]
    w = 4 if cfg == "c1" else 2
    A, B = L_of(sa), L_of(sb)
    rng = np.random.default_rng(3)
    src = O.pack(A, gen.random_bits(rng, 1 << A.d_out, w))
    ref = O.convert(A, B, src)
    for threads in (0, 1):
        got = OC.convert(A.cols, B.cols, A.d_out, w, src, threads=threads).view(ref.dtype)
        assert np.array_equal(got, ref)
    # a sub-range (the bounded samples bench.py times)
    h0 = 37
    n = min(1000, ref.size - h0)
    got = OC.convert(A.cols, B.cols, A.d_out, w, src, h0=h0, n=n).view(ref.dtype)
    assert np.array_equal(got, ref[h0:h0 + n])


def test_convert_broadcast_random():
    """O5 with broadcasting A and B (R1 with zero columns), consistent src."""
    rng = np.random.default_rng(9)
    out_dims = [("i", 3), ("j", 4)]
    hw = [("reg", 3), ("lane", 5), ("warp", 1)]
    for _ in range(10):
        A = L_of(gen.random_distributed(rng, out_dims, hw))
        B = L_of(gen.random_distributed(rng, out_dims, hw))
        T = gen.random_bits(rng, 1 << A.d_out, 4)
        src = O.pack(A, T)
        got = OC.convert(A.cols, B.cols, A.d_out, 4, src).view(src.dtype)
        assert np.array_equal(got, O.convert(A, B, src))


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_gather_matches_numpy_oracle(family):
    L = L_of(W.c4("gather", family, n_i=8, n_j=7))
    rng = np.random.default_rng(1004)
    n = 1 << L.d_in
    src = O.pack(L, gen.random_bits(rng, n, 4))
    idx = O.pack(L, rng.integers(-100, 100, size=n).astype(np.int32))
    ref = O.gather(L, 1, src, idx)
    got = OC.gather(L.cols, L.d_out, 0, 5, 4, src, idx).view(ref.dtype)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_reduce_matches_numpy_oracle(family):
    """O11: fixed-order fp32 bit-equal to numpy's replica; fp64 equal to its fp64 sum."""
    L = L_of(W.c4("reduce", family, n_i=8, n_j=8))
    rng = np.random.default_rng(1005)
    T = rng.random(1 << L.d_out, dtype=np.float32)
    T[::128] = 1.0
    T[1::128] *= np.float32(2.0 ** -20)
    src = O.pack(L, T)
    rep = O.reduce_fixed_order_fp32(L, 1, src)
    got = OC.reduce(L.cols, L.d_out, 0, 8, 7, src)
    assert np.array_equal(got.view(np.uint32), rep.view(np.uint32))
    ref = O.reduce_ref_fp64(L, 1, src)
    got64 = OC.reduce(L.cols, L.d_out, 0, 8, 7, src, fp64=True)
    assert np.allclose(got64, ref, rtol=1e-15, atol=0)


def test_reduce_golden_rows():
    """The hand-derived fp32 goldens of reading R-reduce (tests/golden/reduce_order.json)
    through the C++ replica."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "reduce_order.json")))
    L = O.blocked([4, 8], [1, 2], [4, 8], [1, 1], [1, 0])
    rows = np.array([np.array(c["x_in_u"], dtype=np.float64) * 2.0 ** -24 for c in g["cases"]], dtype=np.float32)
    out = OC.reduce(L.cols, L.d_out, 0, 3, 3, O.pack(L, rows.reshape(-1)))
    assert ["%08x" % int(v) for v in out.view(np.uint32)] == [c["expected_hex"] for c in g["cases"]]
