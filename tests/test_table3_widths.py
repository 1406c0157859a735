"""§8(f) N3, Table 3: [512, k] x {f8, f16} tensors moved between memory
(row-major) and the blocked distributed layouts of tests/golden/table3_contiguity.json
(reading G23), in both directions (load: memory -> distributed, store: distributed ->
memory).  CPU: the executed global vector width on the memory side equals Table 3's
Triton-Linear bitwidth for every row, and the simulated schedule equals the oracle.
GPU: bit-exact against the oracle."""
import json
import os

import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import gen

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")
ROWS = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table3_contiguity.json")))["rows"]


def _layouts(r):
    B = ll.ll_layout_blocked(r["shape"], r["size_per_thread"], [4, 8], [4, 1], [1, 0])
    OB = O.blocked(r["shape"], r["size_per_thread"], [4, 8], [4, 1], [1, 0])
    od = B.out_dims
    OM = O.identity_memory(od)
    M = ll.Layout(OM.in_dims, OM.out_dims, OM.bases)
    assert B.cols() == OB.cols
    return M, B, OM, OB


def _ids():
    return ["%dx%d_f%d" % (r["shape"][0], r["shape"][1], 8 * r["dtype_bytes"]) for r in ROWS]


@pytest.mark.parametrize("r", ROWS, ids=_ids())
@pytest.mark.parametrize("direction", ["load", "store"])
def test_table3_vector_width_and_schedule(r, direction):
    M, B, OM, OB = _layouts(r)
    w = r["dtype_bytes"]
    src_l, dst_l, osrc, odst = (M, B, OM, OB) if direction == "load" else (B, M, OB, OM)
    p = ll.ll_plan_convert(src_l, dst_l, w)
    d = p.describe()
    assert d["exec"] == "tile", d
    t = d["tile"]
    v = t["vld"] if direction == "load" else t["vst"]     # the memory side's vector
    assert (1 << v) * w * 8 == r["bits"], (r, direction, t["vld"], t["vst"])
    T = gen.random_bits(np.random.default_rng(456), 1 << osrc.d_out, w)
    src = O.pack(osrc, T)
    got = p.simulate(src, 1 << odst.d_in)
    assert np.array_equal(got, O.convert(osrc, odst, src))


@pytest.mark.gpu
@pytest.mark.parametrize("r", ROWS, ids=_ids())
@pytest.mark.parametrize("direction", ["load", "store"])
def test_table3_gpu_bitexact(r, direction):
    from tests._util import from_device, to_device
    import torch
    M, B, OM, OB = _layouts(r)
    w = r["dtype_bytes"]
    src_l, dst_l, osrc, odst = (M, B, OM, OB) if direction == "load" else (B, M, OB, OM)
    p = ll.ll_plan_convert(src_l, dst_l, w)
    T = gen.random_bits(np.random.default_rng(457), 1 << osrc.d_out, w)
    src = O.pack(osrc, T)
    n = 1 << odst.d_in
    d_dst = torch.zeros(n, dtype={1: torch.uint8, 2: torch.int16}[w], device="cuda")
    ll.ll_convert(to_device(src), d_dst, p)
    assert np.array_equal(from_device(d_dst, w), O.convert(osrc, odst, src))
