"""GPU fuzz: seeded random conversion cases (tests/_fuzz.py: bijective and broadcast
distributed layouts with batch blocks, Def 4.14 memory layouts, offset permutations,
tiles stored to / loaded from memory; 1-8 byte elements; random plan options) through
the C ABI, each bit-exact against the oracle.  Needs a B200."""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import gen
from tests._fuzz import fuzz_case
from tests._util import empty_device, from_device, to_device

pytestmark = pytest.mark.gpu

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def _seeds(default):
    """Seeds of the fuzz cases: the default list, or LL_FUZZ_SEEDS="a-b" for an
    extended run (e.g. the round-end robustness pass)."""
    import os
    e = os.environ.get("LL_FUZZ_SEEDS")
    if not e:
        return default
    a, b = (int(x) for x in e.split("-"))
    return list(range(a, b + 1))


@pytest.mark.parametrize("seed", _seeds([1, 2, 3]))
def test_fuzz_conversions_bitexact(seed):
    import torch
    rng = np.random.default_rng(7000 + seed)
    ran = 0
    for case in range(50):
        kind, la, lb, w, opts = fuzz_case(rng)
        OA, OB = O.Layout(*la), O.Layout(*lb)
        try:
            plan = ll.ll_plan_convert(ll.Layout(*la), ll.Layout(*lb), w, **opts)
        except ll.LLError as e:
            assert "UNSUPPORTED" in str(e), (case, kind, opts, str(e))   # e.g. SHUFFLE forced on an smem map
            continue
        src = O.pack(OA, gen.random_bits(rng, 1 << OA.d_out, w))
        d_dst = empty_device(1 << OB.d_in, w)
        ll.ll_convert(to_device(src), d_dst, plan)
        torch.cuda.synchronize()
        d = plan.describe()
        assert np.array_equal(from_device(d_dst, w), O.convert(OA, OB, src)), \
            (case, kind, w, opts, d["class"], d["exec"], d.get("tile", {}).get("xchg"))
        ran += 1
    assert ran >= 40
