"""GPU parity of the stmatrix / ldmatrix smem round trips (Thm 5.1): the
CUDA path through the C ABI against the CPU oracle, bit-exact.  Needs a B200."""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen
from tests._matrix_cases import MATRIX_CASES
from tests._util import empty_device, from_device, to_device

pytestmark = pytest.mark.gpu

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def _run(sa, sb, w, seed, **opts):
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w, **opts)
    src = O.pack(OA, gen.random_bits(np.random.default_rng(seed), 1 << OA.d_out, w))
    d_dst = empty_device(1 << OB.d_in, w)
    ll.ll_convert(to_device(src), d_dst, plan)
    import torch
    torch.cuda.synchronize()
    return from_device(d_dst, w), O.convert(OA, OB, src), plan.describe()


def _batched(spec, nb):
    """The same tile layout over 2^nb independent tiles (block bits = batch bits)."""
    return {"out": [("b", nb)] + list(spec["out"]), "in": list(spec["in"]) + [("block", [f"b{k}" for k in range(nb)])]}


@pytest.mark.parametrize("case", MATRIX_CASES, ids=[c[0] for c in MATRIX_CASES])
@pytest.mark.parametrize("nb", [0, 7])
def test_matrix_cases_bitexact(case, nb):
    name, sa, sb, w, (want_st, want_ld) = case
    if nb:
        sa, sb = _batched(sa, nb), _batched(sb, nb)
    got, ref, d = _run(sa, sb, w, 11 + nb, sigma="faithful", force_class="SMEM")
    t = d["tile"]
    assert (t["smem_store"], t["smem_load"]) == (want_st, want_ld)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("cfg", ["c2", "c3", "c3b"])
@pytest.mark.parametrize("smem_instr", ["matrix", "vec"])
def test_paper_configs_matrix_vs_vec_bitexact(cfg, smem_instr):
    """Config 2 / 3 under faithful σ (stmatrix for the accumulator / [1,8] side) and
    config 3b under coalesced σ (stmatrix widens the vector to 16 B), each against the
    vectorised-only plan: both bit-exact."""
    sa, sb = {"c2": W.c2(4), "c3": W.c3(2), "c3b": W.c3b(2)}[cfg]
    sigma = "coalesced" if cfg == "c3b" else "faithful"
    got, ref, d = _run(sa, sb, 2, 1002, sigma=sigma, force_class="SMEM", smem_instr=smem_instr)
    t = d["tile"]
    assert ("stmatrix" in t["smem_store"]) == (smem_instr == "matrix")
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("w", [1, 2, 4])
def test_random_layouts_matrix_bitexact(w):
    """Random distributed pairs (R1) with smem_instr = "matrix" (stmatrix / ldmatrix
    wherever the tile divides), both kernel decompositions, 16 tiles each."""
    rng = np.random.default_rng(5000 + w)
    out = [("i", 5), ("j", 5)]
    kinds = set()
    for R in (1, 2, 3):
        hw = [("reg", R), ("lane", 5), ("warp", 5 - R)]
        for case in range(8):
            sa = _batched(gen.random_distributed(rng, out, hw), 4)
            sb = _batched(gen.random_distributed(rng, out, hw), 4)
            sigma = ("faithful", "coalesced")[case % 2]
            got, ref, d = _run(sa, sb, w, case, sigma=sigma, force_class="SMEM", smem_instr="matrix")
            assert np.array_equal(got, ref), (R, case, d["tile"]["smem_store"], d["tile"]["smem_load"])
            kinds.add((d["tile"]["smem_store"], d["tile"]["smem_load"]))
    assert any("matrix" in a + b for a, b in kinds), kinds
